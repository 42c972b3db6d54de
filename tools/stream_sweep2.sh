#!/bin/bash
B=tools/stream_bench
L2=$((16<<20))
echo "# mode 0 depth 1 vs many; 128 KB chunks"
for c in 16384 65536 131072; do for d in 1 2; do [ $((c*d)) -le 200000 ] && timeout 30 $B 0 $c $d $L2 148 1; done; done
echo "# mode 5: several issuing warps"
for w in 2 4 8; do timeout 30 $B 5 16384 2 $L2 148 $w; timeout 30 $B 5 32768 2 $L2 148 $w; done
echo "# mode 3: tensor tiles"
for c in 8192 16384 32768; do for d in 2 4 6; do [ $((c*d)) -le 200000 ] && timeout 30 $B 3 $c $d $L2 148 1; done; done
echo "# mode 4: gather4"
for c in 8192 16384 32768; do for d in 2 4 6; do [ $((c*d)) -le 200000 ] && timeout 30 $B 4 $c $d $L2 148 1; done; done
timeout 30 $B 4 16384 4 $((2<<30)) 148 1
echo "# mode 1 cp.async, 1 KB per thread per slot"
timeout 30 $B 1 65536 3 $L2 148 1
