# kbench span per ring plan: "b:wcb:xkb:xringKB" entries (0 = launcher default)
for cfg in ${CFGS}; do
  IFS=: read b w x r <<< "$cfg"
  out=$(BM_WCB=$w BM_XKB=$x BM_XRING=$r timeout 60 python tools/kbench.py --b $b --iters 100 2>&1 | tail -1)
  echo "b=$b wcb=$w xkb=$x xring=$r :: $(echo "$out" | python -c 'import sys,json
l=sys.stdin.read()
try:
  r=json.loads(l); print("span %.2f us  call %.2f us" % (r["span_us"], r["us_per_call"]))
except Exception: print(l[:150])')"
done
