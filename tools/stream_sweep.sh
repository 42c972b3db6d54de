#!/bin/bash
# In-kernel L2/HBM -> shared-memory streaming rates (tools/stream_bench.cu), one JSON line each.
B=tools/stream_bench
L2=$((16<<20)); HBM=$((2<<30))
for fp in $L2 $HBM; do
  for c in 8192 16384 32768 65536; do for d in 2 3 4 6; do
    [ $((c*d)) -le 200000 ] && timeout 30 $B 0 $c $d $fp 148 1
  done; done
  timeout 30 $B 1 16384 4 $fp 148 1
  timeout 30 $B 1 16384 8 $fp 148 1
  for cs in 2 4 8; do timeout 30 $B 2 32768 4 $fp 144 $cs; timeout 30 $B 2 16384 8 $fp 144 $cs; done
done
# fewer SMs: per-SM rate when L2 is not shared by all
for n in 16 64 128; do timeout 30 $B 0 32768 4 $L2 $n 1; done
