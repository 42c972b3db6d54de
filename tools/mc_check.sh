# multicast kernel: parity tests + spans vs the default path
BM_MC=1 timeout 300 python -m pytest tests/test_gpu_cells.py -x -q 2>&1 | tail -4
echo "== default"; timeout 120 python tools/kbench.py --b ${SPAN_B:-64,128,192,256,384,512} --iters 200 2>&1 | cut -c1-110
echo "== mc"; BM_MC=1 timeout 120 python tools/kbench.py --b ${SPAN_B:-64,128,192,256,384,512} --iters 200 2>&1 | cut -c1-110
for b in ${PB:-256 512}; do rm -f gpurun_out/pm.txt; BM_MC=1 BM_PHASE_DUMP=gpurun_out/pm.txt timeout 60 python tools/kbench.py --b $b --iters 3 >/dev/null 2>&1
echo "== mc phases b=$b"; python tools/phases.py gpurun_out/pm.txt | grep -E "mainloop|setup|bar1|reduce|bar2|stage kb|weight chunk|stage 0|after PDL" ; done
