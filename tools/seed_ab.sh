#!/bin/bash
# A/B of the landmark seeding (reading R9): the paper's sampler alone
# (SKNN_SEEDING=paper) vs the default (D^2 split for dp >= 16); bench lines.
out=gpurun_out/${1:-seed_ab}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
for c in C3 C5 C3int C2; do
  for sd in default paper; do
    if [ $sd = paper ]; then export SKNN_SEEDING=paper; else unset SKNN_SEEDING; fi
    timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | \
      python -c "import json,sys; r=json.loads(sys.stdin.readline()); print(json.dumps({'config':'$c','seeding':'$sd','ms':r['ms_per_step'],'pruned':r.get('pruned_pct')}))" >> $out/seed_ab.jsonl
  done
done
unset SKNN_SEEDING
cat $out/seed_ab.jsonl
