# Round-end validation bundle on the final code (TAG): GPU tests, smoke, bench lines
# configs[1]/[2]/[3], launch list, full capture of the dominant kernel.
T=${TAG:-r1i}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/tests_$T.log
timeout 200 python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" >> gpurun_out/tests_$T.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_lstm_$T.json 2> gpurun_out/bench_lstm_$T.err
timeout 600 python bench.py --workload seq2seq > gpurun_out/bench_seq2seq_$T.json 2> gpurun_out/bench_seq2seq_$T.err
timeout 600 python bench.py --workload tree > gpurun_out/bench_tree_$T.json 2> gpurun_out/bench_tree_$T.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$T.json 2> gpurun_out/bench_ref_$T.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$T.csv \
  python bench.py --steps 2 --warmup 1 --reqs 2000 --rate 100000 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_$T.csv > gpurun_out/launches_summary_$T.txt 2>&1
