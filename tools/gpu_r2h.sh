timeout 120 python tools/pair_cmp.py gpurun_out/pc_new.npz 2>&1 | tail -2
BM_PAIR2=0 timeout 120 python tools/pair_cmp.py gpurun_out/pc_old.npz gpurun_out/pc_new.npz 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_cells.py -x -q 2>&1 | tail -5
timeout 300 python tools/kbench.py --cell lstm --b 64,129,192,256,320,384,448,512 --iters 100 > gpurun_out/kb_pair2.log 2>&1
python tools/kb_table.py gpurun_out/kb_pair2.log
for b in 336 512; do rm -f gpurun_out/ph2_$b.txt; BM_PHASE_DUMP=gpurun_out/ph2_$b.txt timeout 100 python tools/kbench.py --b $b --iters 3 > /dev/null 2>&1; python tools/phases.py gpurun_out/ph2_$b.txt | head -12; done
timeout 600 python tools/s2s_one.py 20000 20000 1468 2>&1 | tail -2
