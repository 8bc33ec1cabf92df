python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for pass in 1 2; do for c in C2 C3 C5; do for v in default nosplit; do
  if [ $v = nosplit ]; then export SKNN_SPLIT=0; else unset SKNN_SPLIT; fi
  timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | python3 -c "import json,sys; r=json.loads(sys.stdin.readline()); print(\"$c $v\", round(r[\"ms_per_step\"],4), {k: round(x,3) for k,x in r[\"stage_ms\"].items()})"
done; done; done
