timeout 300 python -m pytest tests/test_gpu_cells.py -x -q 2>&1 | tail -2
BM_PAIR=0 BM_PCHUNK=64 timeout 300 python -m pytest tests/test_gpu_cells.py -x -q -k "lstm_step or tree or invariance_bitwise" 2>&1 | tail -2
echo "== default"; BS=128,256,384,512 timeout 200 python tools/dual_bench.py 2>&1
for cfg in "64 1 32" "64 2 32" "128 1 32"; do set -- $cfg; echo "== pchunk=$1 wcb=$2 xring=$3"; BM_PAIR=0 BM_PCHUNK=$1 BM_WCB=$2 BM_XRING=$3 BS=128,256,384,512 timeout 200 python tools/dual_bench.py 2>&1; done
