# Round profiling bundle (one gpurun call, 1 GPU). TAG=r1c
T=${TAG:-r1c}
timeout 600 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$T.csv \
  python bench.py --steps 2 --warmup 1 --reqs 2000 --rate 100000 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_$T.csv > gpurun_out/launches_summary_$T.txt 2>&1
for k in cell_pair_kernel cell_step_sm100_kernel; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 200 -c 3 -o gpurun_out/prof_${k}_$T \
    python bench.py --steps 1 --warmup 1 --reqs 3000 --rate 600000 --no-cpu-baseline > gpurun_out/ncu_${k}_$T.log 2>&1
  ncu -i gpurun_out/prof_${k}_$T.ncu-rep --page raw --csv > gpurun_out/prof_${k}_${T}_raw.csv 2>/dev/null
done
