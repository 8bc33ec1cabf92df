#!/bin/bash
# A/B timing of library variants on the GPU box (run under gpurun):
#   tools/ab_run.sh <tag> <configs> <variant>...   (variant "cur" = in-tree build, else abl/<variant>.so)
tag=$1; cfgs=$2; shift 2
out=gpurun_out/$tag; mkdir -p $out
for pass in 1 2; do
  for v in "$@"; do
    if [ $v = cur ]; then L=; else L=abl/$v.so; fi
    SKNN_LIB=$L timeout 600 python tools/sweep.py --configs $cfgs --reps 5 --variants ${SWEEP_VARIANTS:-default} > $out/${v}_$pass.jsonl 2>&1
  done
done
for f in $out/*.jsonl; do
  python - "$f" <<'PY'
import json, sys
f = sys.argv[1]
for l in open(f):
    try:
        d = json.loads(l)
    except Exception:
        continue
    print("%-22s %-14s %-5s %8.3f  %s ins/q %.1f evals/q %.0f" % (f.split("/")[-1], d["variant"][:14], d["config"], d["ms_total"],
          {k: round(v, 3) for k, v in d["stages"].items() if v}, d["inserts_per_query"], d["evals_per_query"]))
PY
done
