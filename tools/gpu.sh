#!/bin/bash
# GPU-side runs of this repo, one entry point (run under gpurun from the repo root):
#
#   bash tools/gpu.sh full      [TAG]   smoke + pytest -m gpu + default bench.py (round-end set)
#   bash tools/gpu.sh profile   [TAG]   ncu launch lists + full captures inside the bench workloads,
#                                       per-class traffic -> gpurun_out/traffic_<wl>.json
#   bash tools/gpu.sh kbench    [TAG]   per-b device spans of every cell kernel (tools/kbench.py)
#   bash tools/gpu.sh phases    [TAG]   BM_PHASE_DUMP phase timelines of LSTM steps (tools/phases.py)
#   bash tools/gpu.sh stream            in-kernel L2/HBM -> shared streaming rates (tools/stream_bench.cu)
#   bash tools/gpu.sh sanitize          compute-sanitizer memcheck / synccheck / racecheck over the cell kernels
#   bash tools/gpu.sh sweep     [TAG]   kbench of one cell under each env plan in $PLANS (';'-separated,
#                                       e.g. PLANS='BM_PAIR_XKB=1;BM_PAIR_WCPA=0 BM_PAIR_WS=4'), CELL, BS
#
# Outputs go to gpurun_out/ (merged back by gpurun); copy what is to be judged to profiles/.
set -u
CMD=${1:-full}
TAG=${2:-r2}
mkdir -p gpurun_out
case "$CMD" in
full)
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc $?"
  timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.log 2>&1; echo "tests rc $?"
  tail -3 gpurun_out/tests_$TAG.log
  grep -o "AssertionError.*" gpurun_out/tests_$TAG.log | head -3
  timeout 1500 python bench.py --steps 5 --warmup 2 --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1
  echo "bench rc $?"
  python tools/bench_summary.py gpurun_out/bench_$TAG.json
  ;;
profile)
  # bench.py at a fixed offered rate near lambda* with fewer requests (serialised ncu passes);
  # spec: workload, rate, requests, launches to skip (burst calibration x 2 + warm-up step)
  for spec in "lstm 540000 20000 3900" "seq2seq 40000 2000 8000" "tree 65000 10000 27000"; do
    set -- $spec; wl=$1; R=$2; N=$3; SK=$4
    B="python bench.py --workload $wl --rate $R --reqs $N --steps 1 --warmup 1 --no-cpu-baseline --extra none"
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s $SK -c 3000 --csv \
      --log-file gpurun_out/launches_${wl}_$TAG.csv $B > /dev/null 2>&1
    timeout 1200 ncu --set full --clock-control none --import-source on -k regex:cell_ -s $SK -c 12 \
      -o gpurun_out/prof_${wl}_$TAG $B > gpurun_out/ncu_${wl}_$TAG.log 2>&1
    ncu -i gpurun_out/prof_${wl}_$TAG.ncu-rep --page raw --csv > gpurun_out/prof_${wl}_${TAG}_raw.csv 2>/dev/null
    python tools/traffic_classes.py gpurun_out/prof_${wl}_${TAG}_raw.csv gpurun_out/launches_${wl}_$TAG.csv \
      gpurun_out/traffic_${wl}.json "$B" > /dev/null
    echo "$wl profiled"
  done
  ;;
kbench)
  for c in lstm leaf internal proj; do
    timeout 300 python tools/kbench.py --cell $c --b 1,16,32,64,128,192,256,320,384,448,512 --iters 100 \
      > gpurun_out/kbench_${c}_$TAG.log 2>&1
    python tools/kb_table.py gpurun_out/kbench_${c}_$TAG.log
  done
  ;;
phases)
  for b in ${B_LIST:-64 256 384 512}; do
    rm -f gpurun_out/ph_${b}_$TAG.txt
    BM_PHASE_DUMP=gpurun_out/ph_${b}_$TAG.txt timeout 100 python tools/kbench.py --b $b --iters 3 > /dev/null 2>&1
    echo "== b=$b"
    python tools/phases.py gpurun_out/ph_${b}_$TAG.txt 2>&1 | tail -16
    if [ $b -gt 128 ]; then python tools/pair_phases.py gpurun_out/ph_${b}_$TAG.txt 2>&1; fi
  done
  ;;
stream)
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/stream_bench tools/stream_bench.cu
  S=tools/stream_bench; L2=$((16 << 20)); HBM=$((2 << 30))
  for fp in $L2 $HBM; do for c in 16384 32768 65536; do timeout 30 $S 0 $c 2 $fp 148 1; done; done
  for G in 1 2 4; do timeout 30 $S 7 16384 2 $L2 148 $G; done          # cp.async, G thread groups
  for G in 2 4; do timeout 30 $S 8 16384 2 $L2 148 $G; done            # TMA bulk, G issuing lanes
  for c in 16384 32768; do timeout 30 $S 3 $c 4 $L2 148 1; timeout 30 $S 4 $c 4 $L2 148 1; done  # tensor / gather4
  ;;
sweep)
  IFS=';' read -ra PL <<< "${PLANS:-}"
  for plan in "" "${PL[@]}"; do
    echo "== plan: ${plan:-default}"
    env $plan timeout 300 python tools/kbench.py --cell ${CELL:-lstm} --b ${BS:-192,256,384,512} --iters 200 \
      > gpurun_out/sweep_tmp.log 2>&1
    python tools/kb_table.py gpurun_out/sweep_tmp.log
    grep -i "error\|Traceback" gpurun_out/sweep_tmp.log | head -3
  done > gpurun_out/sweep_$TAG.log 2>&1
  cat gpurun_out/sweep_$TAG.log
  ;;
sanitize)
  S=/usr/local/cuda/bin/compute-sanitizer
  for tool in memcheck synccheck racecheck; do
    echo "== $tool: tools/memcheck_small.py (single-CTA cells, Seq2Seq, tree)"
    timeout 900 $S --tool $tool --print-limit 10 python tools/memcheck_small.py 2>&1 | grep -v "^\s*$" | tail -6
    echo "== $tool: tools/pair_cmp.py (CTA-pair kernel, b = 129..512)"
    timeout 900 $S --tool $tool --print-limit 10 python tools/pair_cmp.py /tmp/pc.npz 2>&1 | grep -v "^\s*$" | tail -6
  done
  ;;
*)
  echo "usage: bash tools/gpu.sh full|profile|kbench|phases|stream|sanitize [TAG]"; exit 2 ;;
esac
