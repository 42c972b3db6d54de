for b in ${B_LIST:-1 64 336 512}; do
  rm -f gpurun_out/ph_$b.txt
  BM_PHASE_DUMP=gpurun_out/ph_$b.txt timeout 100 python tools/kbench.py --b $b --iters 3 > /dev/null 2>&1
  echo "== b=$b"
  python tools/phases.py gpurun_out/ph_$b.txt 2>&1 | tail -18
  if [ $b -gt 128 ]; then python tools/pair_phases.py gpurun_out/ph_$b.txt 2>&1 | tail -20; fi
done
