#!/bin/bash
# compute-sanitizer evidence: memcheck, racecheck and
# synccheck over small joins that reach every kernel family (build, level-1,
# warp-union scan with split tasks, warp-per-query scan, big-k, partial filter,
# exact + split-precision dense tiles, merge). Run under gpurun:
#   tools/sanitize.sh <tag>   -> gpurun_out/<tag>/san_<tool>_<case>.txt
out=gpurun_out/${1:-san}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
CS=/usr/local/cuda/bin/compute-sanitizer
run() {  # run <tool> <name> <args...>
  local tool=$1 name=$2; shift 2
  timeout 900 $CS --tool $tool --error-exitcode 7 --print-limit 20 python "$@" > $out/san_${tool}_$name.txt 2>&1
  echo "$tool $name rc=$? $(grep -c 'ERROR SUMMARY: 0 errors\|RACECHECK SUMMARY: 0 hazards' $out/san_${tool}_$name.txt) $(grep 'SUMMARY' $out/san_${tool}_$name.txt | tail -1)"
}
for tool in memcheck racecheck synccheck; do
  run $tool c1 tools/run_one.py C1 1.0 1
  run $tool c2 tools/run_one.py C2 0.02 1
  run $tool c4_auto tools/run_one.py C4 0.003 1
  run $tool c4_dense tools/run_one.py C4 0.003 1 force_path=dense
  run $tool c5 tools/run_one.py C5 0.0015 1
  run $tool c3_partial tools/run_one.py C3 0.03 1 force_path=partial
  run $tool c3_bigk tools/run_one.py C3 0.03 1 knn_k=200
  run $tool merge tools/merge_bench.py --nq 5000 --k 32 --P 3,8 --reps 1
done
