# phase summary of direct steps under ring plans: CFGS="wcb:xringKB ..." B=...
for cfg in ${CFGS:-0:0}; do
  w=${cfg%%:*}; x=${cfg##*:}
  rm -f gpurun_out/phc_$w_$x.txt
  BM_WCB=$w BM_XRING=$x BM_EXPERIMENT=${X:-0} BM_PHASE_DUMP=gpurun_out/phc_$w_$x.txt timeout 100 python tools/kbench.py --cell ${CELL:-lstm} --b ${B:-256} --iters 3 > /dev/null
  echo "== wcb=$w xring=$x exp=${X:-0}"; python tools/phases.py gpurun_out/phc_$w_$x.txt | grep -E "^step|stage kb|weight chunk at|mainloop|reduce|bar1|row table|SM clock" | tail -8
done
