timeout 900 python -m pytest tests/test_gpu_cells.py -x -q 2>&1 | tail -2
for c in leaf proj internal lstm; do
  timeout 300 python tools/kbench.py --cell $c --b 1,16,64,128 --iters 100 > gpurun_out/kb_new_$c.log 2>&1; echo "== new $c"; python tools/kb_table.py gpurun_out/kb_new_$c.log
done
BM_PROJ_TMA=0 timeout 300 python tools/kbench.py --cell proj --b 1,16,64,128 --iters 100 > gpurun_out/kb_old_proj.log 2>&1; echo "== old proj"; python tools/kb_table.py gpurun_out/kb_old_proj.log
BM_WSLOTS=1 timeout 300 python tools/kbench.py --cell lstm --b 1,16,64,128 --iters 100 > gpurun_out/kb_old_lstm.log 2>&1; echo "== 1 lane lstm"; python tools/kb_table.py gpurun_out/kb_old_lstm.log
