timeout 300 compute-sanitizer --tool memcheck --print-limit 3 python tools/pair_cmp.py /tmp/x.npz 2>&1 | head -60
