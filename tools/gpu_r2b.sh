set -x
bash tools/stream_sweep.sh > gpurun_out/stream_r2b.log 2>&1
timeout 900 python tools/s2s_diag.py 4000 > gpurun_out/s2s_diag_r2b.log 2>&1; echo diag rc $?
tail -40 gpurun_out/s2s_diag_r2b.log
