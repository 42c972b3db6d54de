timeout 300 python -m pytest tests/test_gpu_cells.py -x -q -k "pair or 300 or 512" 2>&1 | tail -2
timeout 120 python tools/kbench.py --b 257,320,384,448,512 --iters 200 2>&1 | cut -c1-100
for b in 384 512; do rm -f gpurun_out/pe.txt; BM_PHASE_DUMP=gpurun_out/pe.txt timeout 60 python tools/kbench.py --b $b --iters 3 >/dev/null 2>&1
echo "== phases b=$b"; python tools/pair_phases.py gpurun_out/pe.txt | head -7; done
