BM_MC=2 timeout 300 python -m pytest tests/test_gpu_cells.py -x -q -k "not invariance" 2>&1 | tail -2
for C in 2 4 8; do echo "== mc2 C=$C"; BM_MC=2 BM_MC_C=$C timeout 120 python tools/kbench.py --b ${SPAN_B:-64,128,256,384,512} --iters 200 2>&1 | cut -c1-100; done
for b in ${PB:-256 512}; do rm -f gpurun_out/pm.txt; BM_MC=2 BM_PHASE_DUMP=gpurun_out/pm.txt timeout 60 python tools/kbench.py --b $b --iters 3 >/dev/null 2>&1
echo "== mc2 phases b=$b"; python tools/phases.py gpurun_out/pm.txt | tail -14 | grep -E "mainloop|setup|bar1|reduce|bar2|stage kb|stage 0|after PDL" ; done
