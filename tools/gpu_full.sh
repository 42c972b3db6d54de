# full GPU suite + smoke + default bench (round-end equivalent); TAG names the outputs
TAG=${TAG:-r2}
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc $?
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/tests_$TAG.log 2>&1; echo tests rc $?
tail -4 gpurun_out/tests_$TAG.log
grep -o "AssertionError.*" gpurun_out/tests_$TAG.log | head -3
timeout 1200 python bench.py --steps 5 --warmup 2 --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1; echo bench rc $?
python tools/bench_summary.py gpurun_out/bench_$TAG.json
