# compute-sanitizer over the smoke path (configs[0] chain, one h=1024 Seq2Seq with <eos>-free
# decode, one 16-leaf tree) and a small h=1024 chain trace: memcheck, racecheck, synccheck.
for tool in memcheck racecheck synccheck; do
  echo "== $tool"
  timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 \
    python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | grep -E "ERROR SUMMARY|smoke ok|Error|error|hazard" | head -20
done
