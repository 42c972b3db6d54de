# final validation bundle: GPU tests, smoke, bench line, launch list (TAG)
T=${TAG:-r1e}
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/tests_$T.log
timeout 200 python -c "import __graft_entry__ as g; g.build(); g.smoke()" >> gpurun_out/tests_$T.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$T.csv \
  python bench.py --steps 2 --warmup 1 --reqs 2000 --rate 100000 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_$T.csv > gpurun_out/launches_summary_$T.txt 2>&1
