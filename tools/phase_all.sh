# Phase timelines (BM_PHASE_DUMP) + kbench spans of the LSTM cell step at several b.
# usage: B_LIST="64 256 384 512" bash tools/phase_all.sh
for b in ${B_LIST:-64 256 384 512}; do
  rm -f gpurun_out/ph_$b.txt
  BM_PHASE_DUMP=gpurun_out/ph_$b.txt timeout 100 python tools/kbench.py --b $b --iters 3 > /dev/null 2>&1
  echo "== b=$b"
  python tools/phases.py gpurun_out/ph_$b.txt 2>&1 | tail -16
  if [ $b -gt 256 ]; then python tools/pair_phases.py gpurun_out/ph_$b.txt 2>&1; fi
done
timeout 200 python tools/kbench.py --b ${SPAN_B:-16,64,128,192,256,320,384,448,512} --iters 200 2>&1 | tail -12
