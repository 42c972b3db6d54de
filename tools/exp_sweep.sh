# phase dumps of direct cell steps under the diagnostic BM_EXPERIMENT bits
for x in ${XS:-0 1 2 8 9}; do
  rm -f gpurun_out/phx_$x.txt
  BM_EXPERIMENT=$x BM_PHASE_DUMP=gpurun_out/phx_$x.txt timeout 100 python tools/kbench.py --b ${B:-256} --iters 3 > /dev/null
  echo "== experiment=$x"; python tools/phases.py gpurun_out/phx_$x.txt | grep -E "^step|stage kb|weight chunk at|mainloop|reduce|bar1|row table|first hand" | tail -8
done
