# per-task device cost (taskbench) under ring plans: CFGS="wcb:xringKB ..." (0:0 = default)
for cfg in ${CFGS:-0:0 4:32 4:16 2:16 1:32}; do
  w=${cfg%%:*}; x=${cfg##*:}
  echo "== wcb=$w xring=$x"
  BM_WCB=$w BM_XRING=$x BM_TIME_EVERY=100000000 timeout 120 python tools/taskbench.py --persistent 0 --b ${B:-16,64,128} --steps 96 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()); continue
    print('  b=%4d us/task %6.2f' % (r['b'], r['us_per_task']))"
done
