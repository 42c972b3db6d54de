for cfg in "0 0" "2 64" "2 96" "2 128" "1 128" "1 160" "4 64" "4 96"; do
  set -- $cfg
  echo "== wcb=$1 xring=$2"
  BM_WCB=$1 BM_XRING=$2 timeout 120 python tools/kbench.py --b 16,64,128,256,512 --iters 300 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()); continue
    print('  b=%4d us/call %6.2f span %6.2f' % (r['b'], r['us_per_call'], r['span_us']))"
done
