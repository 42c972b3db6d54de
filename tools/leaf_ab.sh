# Leaf split-K A/B (BM_LEAF_S = 2: 512-wide K slices, 64 CTAs; 4: 256-wide, 128 CTAs)
T=${TAG:-r1j}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cells.py tests/test_gpu_engine.py -q -x -k "tree or leaf" 2>&1 | tail -5 > gpurun_out/leaf_tests_$T.log
for s in 2 4; do
  BM_LEAF_S=$s timeout 300 python tools/kbench.py --cell leaf --b 1,16,64,128,256,512 > gpurun_out/leaf_kbench_S${s}_$T.txt 2>&1
done
for rep in 1 2; do for s in 2 4; do
  BM_LEAF_S=$s timeout 600 python bench.py --workload tree > gpurun_out/bench_tree_S${s}_${rep}_$T.json 2> gpurun_out/bench_tree_S${s}_${rep}_$T.err
done; done
