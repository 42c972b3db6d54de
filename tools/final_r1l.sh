# Final round-1 check on the final code (leaf S = 4 included): full GPU suite, smoke, default
# bench line, tree bench line; then internal-cell plan experiments for the next round.
T=${TAG:-r1l}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -5 > gpurun_out/tests_$T.log
timeout 200 python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" >> gpurun_out/tests_$T.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_lstm_$T.json 2> gpurun_out/bench_lstm_$T.err
timeout 600 python bench.py --workload tree > gpurun_out/bench_tree_$T.json 2> gpurun_out/bench_tree_$T.err
for cfg in "" "BM_XKB=2" "BM_WCB=2" "BM_XRING=16" "BM_XRING=32" "BM_WCB=1"; do
  echo "== $cfg" >> gpurun_out/internal_plans_$T.txt
  env $cfg timeout 300 python tools/kbench.py --cell internal --b 1,16,32,64 >> gpurun_out/internal_plans_$T.txt 2>&1
done
