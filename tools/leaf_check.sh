# leaf xkb plan: parity + invariance, kbench, tree bench (TAG)
T=${TAG:-r1p}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cells.py tests/test_gpu_engine.py -q -x -k "tree or leaf or internal" 2>&1 | tail -5 > gpurun_out/leaf_tests_$T.log
timeout 300 python tools/kbench.py --cell leaf --b 1,16,32,64,65,128,129,256,512 > gpurun_out/leaf_kbench_$T.txt 2>&1
for rep in 1 2; do
  timeout 600 python bench.py --workload tree > gpurun_out/bench_tree_${rep}_$T.json 2> gpurun_out/bench_tree_${rep}_$T.err
done
