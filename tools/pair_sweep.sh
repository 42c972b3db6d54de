# kbench span of the CTA-pair kernel per plan: "b:S:wcb:xkb" (0 = launcher default)
for cfg in ${CFGS}; do
  IFS=: read b S w x <<< "$cfg"
  out=$(BM_PAIR_S=$S BM_PAIR_WCB=$w BM_PAIR_XKB=$x timeout 60 python tools/kbench.py --b $b --iters 100 2>&1 | tail -1)
  echo "b=$b S=$S wcb=$w xkb=$x :: $(echo "$out" | python -c 'import sys,json
l=sys.stdin.read()
try:
  r=json.loads(l); print("span %.2f us  call %.2f us" % (r["span_us"], r["us_per_call"]))
except Exception: print(l[:150])')"
done
