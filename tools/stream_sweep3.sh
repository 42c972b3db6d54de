B=tools/stream_bench; L2=$((16<<20))
for G in 1 2 4 8; do for c in 8192 16384; do timeout 30 $B 7 $c 2 $L2 148 $G; done; done
timeout 30 $B 7 32768 2 $L2 148 2
timeout 30 $B 7 32768 1 $L2 148 4
for G in 2 4; do timeout 30 $B 8 16384 2 $L2 148 $G; timeout 30 $B 8 32768 2 $L2 148 $G; done
