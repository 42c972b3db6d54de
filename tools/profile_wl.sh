# Launch list + one full capture of sampled cell-step launches for configs[2] / configs[3] (TAG)
T=${TAG:-r1k}
mkdir -p gpurun_out
for wl in seq2seq tree; do
  if [ $wl = seq2seq ]; then R=40000; N=600; else R=60000; N=3000; fi
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches_${wl}_$T.csv \
    python bench.py --workload $wl --steps 2 --warmup 1 --reqs $N --rate $R --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:cell_ -s 400 -c 12 -o gpurun_out/prof_${wl}_$T \
    python bench.py --workload $wl --steps 1 --warmup 1 --reqs $N --rate $R --no-cpu-baseline > gpurun_out/ncu_${wl}_$T.log 2>&1
  ncu -i gpurun_out/prof_${wl}_$T.ncu-rep --page raw --csv > gpurun_out/prof_${wl}_${T}_raw.csv 2>/dev/null
  python tools/traffic_wl.py $T $wl gpurun_out/traffic_${wl}_$T.json > /dev/null 2> gpurun_out/traffic_${wl}_$T.err
done
