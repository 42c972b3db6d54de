set -x
timeout 120 python tools/pair_cmp.py gpurun_out/pc_new.npz
BM_PAIR2=0 timeout 120 python tools/pair_cmp.py gpurun_out/pc_old.npz gpurun_out/pc_new.npz
timeout 900 python -m pytest tests/test_gpu_cells.py -x -q 2>&1 | tail -5
timeout 300 python tools/kbench.py --cell lstm --b 64,129,192,256,320,384,448,512 --iters 100 > gpurun_out/kb_pair2.log 2>&1
BM_PAIR2=0 timeout 300 python tools/kbench.py --cell lstm --b 129,192,256,320,384,448,512 --iters 100 > gpurun_out/kb_pair1.log 2>&1
for f in kb_pair2 kb_pair1; do python -c "
import json
for l in open('gpurun_out/$f.log'):
    if l.startswith('{'):
        d=json.loads(l); ks=[k for k in d if k.startswith('k')]
        print('$f', d['b'], round(d['us_per_call'],2), [(k, round(d[k]['span_us'],2), round(d[k]['TFLOPs'],0)) for k in ks])
"; done
for b in 336 512; do rm -f gpurun_out/ph2_$b.txt; BM_PHASE_DUMP=gpurun_out/ph2_$b.txt timeout 100 python tools/kbench.py --b $b --iters 3 > /dev/null 2>&1; done
B=tools/stream_bench; L2=$((16<<20))
for c in 16384 32768 49152; do timeout 30 $B 6 $c 4 $L2 148 1; timeout 30 $B 1 $c 4 $L2 148 1; done
timeout 600 python tools/s2s_one.py 20000 20000 1468,5,77 > gpurun_out/s2s_one_r2g.log 2>&1; cat gpurun_out/s2s_one_r2g.log | tail -5
