set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_r2a.log 2>&1; echo smoke rc $?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/tests_r2a.log 2>&1; echo tests rc $?
tail -5 gpurun_out/tests_r2a.log
timeout 900 python bench.py --steps 5 --warmup 2 --out gpurun_out/bench_r2a.json > gpurun_out/bench_r2a.log 2>&1; echo bench rc $?
tail -c 600 gpurun_out/bench_r2a.log
for c in lstm leaf internal proj; do timeout 300 python tools/kbench.py --cell $c --b 1,16,32,64,128,192,256,320,384,448,512 --iters 100 > gpurun_out/kbench_${c}_r2a.log 2>&1; done
echo done
