# main-loop phase under diagnostic experiment bits (single-CTA kernel): B, XS
for b in ${BS:-64 256}; do
for x in ${XS:-0 1 2 3 6 8}; do
  rm -f gpurun_out/px.txt
  BM_PAIR=0 BM_EXPERIMENT=$x BM_PHASE_DUMP=gpurun_out/px.txt timeout 100 python tools/kbench.py --b $b --iters 3 > /dev/null 2>&1
  echo "== b=$b exp=$x"; python tools/phases.py gpurun_out/px.txt | grep -E "mainloop|reduce|bar1|stage kb|weight chunk at|stage 0 issued" | tail -6
done; done
