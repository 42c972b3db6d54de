BM_WCPA_MIN=64 timeout 300 python -m pytest tests/test_gpu_cells.py -x -q -k "lstm_step_parity or stack" 2>&1 | tail -2
for nb in 4 2; do echo "== wcpa blocks=$nb"; BM_WCPA_MIN=64 BM_WCPA_BLOCKS=$nb timeout 120 python tools/kbench.py --b ${SPAN_B:-64,128,192,256,320,384,448,512} --iters 200 2>&1 | cut -c1-100; done
for b in ${PB:-256 512}; do rm -f gpurun_out/pw.txt; BM_WCPA_MIN=64 BM_PHASE_DUMP=gpurun_out/pw.txt timeout 60 python tools/kbench.py --b $b --iters 3 >/dev/null 2>&1
echo "== wcpa phases b=$b"; python tools/pair_phases.py gpurun_out/pw.txt; done
