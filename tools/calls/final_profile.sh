#!/bin/bash
# Round-2 evidence pass (gpurun, one GPU): bench lines for every config, the
# reference arm, the ncu launch list of the bench command, ncu --set full of
# every config's dominant kernels (reduced to raw CSV + markdown + hot lines).
tag=${1:-r02final}
out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
source tools/ncu_reduce.sh
KEEP=""
timeout 600 python bench.py > $out/bench_C2.jsonl 2> $out/bench_C2.err
for c in C1 C3 C4 C5; do timeout 600 python bench.py --config $c --no-cpu-baseline > $out/bench_$c.jsonl 2> $out/bench_$c.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $out/bench_C2_ref.jsonl 2> $out/bench_C2_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_C2.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $out/launches_C2.txt 2>&1
NCU="ncu --set full --import-source on --clock-control none -c 1"
prof() {  # prof <name> <kernel regex> <run_one args...>
  local name=$1 kre=$2; shift 2
  timeout 900 $NCU -k regex:"$kre" -o $out/$name python tools/run_one.py "$@" > $out/$name.txt 2>&1
  reduce $out/$name
}
prof c2_k_scan_tpq '^k_scan_tpq$' C2 1.0 2
prof c2_k_level1 '^k_level1$' C2 1.0 2
prof c3_k_scan_tpq '^k_scan_tpq$' C3 1.0 2
prof c4_k_scan_wpq '^k_scan_wpq$' C4
prof c4_k_dense_exact '^k_dense_exact$' C4
prof c4_k_dense_exact_alldense '^k_dense_exact$' C4 1.0 1 force_path=dense
prof c4_k_assign_tc '^k_assign_tc$' C4
prof c5_k_scan_tpq '^k_scan_tpq$' C5
prof c5_k_assign_tc '^k_assign_tc$' C5
prof c5_k_level1 '^k_level1$' C5
timeout 900 $NCU -k regex:"^k_merge" -o $out/merge_p8 python tools/merge_bench.py --reps 1 > $out/merge_ncu.txt 2>&1; reduce $out/merge_p8
timeout 300 python tools/merge_bench.py --P 2,4,8 > $out/merge_bench.jsonl 2>&1
for f in $out/*.md; do tail -1 $f | cut -c1-200; done
for c in C2 C1 C3 C4 C5; do cut -c1-300 $out/bench_$c.jsonl; done
