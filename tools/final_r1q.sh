# Round-1 closing check on the final code: full GPU suite, smoke, default bench line (TAG)
T=${TAG:-r1q}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -5 > gpurun_out/tests_$T.log
timeout 200 python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" >> gpurun_out/tests_$T.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_lstm_$T.json 2> gpurun_out/bench_lstm_$T.err
