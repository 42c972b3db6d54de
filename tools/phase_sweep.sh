# phase dumps of direct cell steps under a few ring plans (BM_WCB / BM_XRING)
for cfg in "0 0" "4 64"; do
  set -- $cfg
  rm -f gpurun_out/ph_$1_$2.txt
  BM_WCB=$1 BM_XRING=$2 BM_PHASE_DUMP=gpurun_out/ph_$1_$2.txt timeout 100 python tools/kbench.py --b ${B:-16,256} --iters 6 > /dev/null
  echo "== wcb=$1 xring=$2"; python tools/phases.py gpurun_out/ph_$1_$2.txt | grep -v "^  [a-z]* *us: min" 
done
