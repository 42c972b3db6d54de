# leaf cell: K blocks per activation hand-off (BM_XKB) sweep (TAG)
T=${TAG:-r1o}
mkdir -p gpurun_out
for cfg in "" "BM_XKB=2" "BM_XKB=4" "BM_XKB=2 BM_XRING=64" "BM_XKB=4 BM_XRING=64"; do
  echo "== $cfg" >> gpurun_out/leaf_plans_$T.txt
  env $cfg timeout 300 python tools/kbench.py --cell leaf --b 1,16,32,64,128,256 >> gpurun_out/leaf_plans_$T.txt 2>&1
done
