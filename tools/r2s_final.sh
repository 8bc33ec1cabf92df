#!/bin/bash
# End-of-session evidence pass (run under gpurun, one GPU):
#   tools/r2s_final.sh <tag>
# -> gpurun_out/<tag>/: GPU test log, bench lines C1-C5 (C2 with cpu_baseline),
#    the reference arm, the C2 bench's ncu launch list, ncu --set full of the C2
#    scan, of the dense-only kernel (dorothea shape) and live timelines.
tag=${1:-final}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.txt 2>&1 || { tail $out/build.txt; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q > $out/pytest_gpu.txt 2>&1; echo "pytest rc=$?"; tail -2 $out/pytest_gpu.txt
timeout 600 python bench.py > $out/bench_C2.jsonl 2> $out/bench_C2.err
for c in C1 C3 C4 C5; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > $out/bench_$c.jsonl 2> $out/bench_$c.err
done
timeout 900 python bench.py --impl reference > $out/bench_C2_ref.jsonl 2> $out/bench_C2_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_C2.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $out/ncu_launch.txt 2>&1
NCU="ncu --set full --import-source on --clock-control none -c 1"
timeout 900 $NCU -k regex:"^k_scan_tpq" -o $out/c2_k_scan_tpq python tools/run_one.py C2 1.0 2 > $out/ncu_c2.txt 2>&1
timeout 900 $NCU -k regex:"^k_brute_tiled" -o $out/dor_k_brute_tiled python tools/run_one.py DOR 1.0 1 > $out/ncu_dor.txt 2>&1
timeout 900 $NCU -k regex:"^k_dense_exact" -o $out/c4_k_dense_exact python tools/run_one.py C4 1.0 1 > $out/ncu_c4d.txt 2>&1
for r in c2_k_scan_tpq dor_k_brute_tiled c4_k_dense_exact; do
  [ -f $out/$r.ncu-rep ] || continue
  python profiles/ncu_summary.py $out/$r.ncu-rep $r > $out/$r.md 2>/dev/null
  python tools/ncu_lines.py $out/$r.ncu-rep 40 > $out/$r.lines.txt 2>/dev/null
  rm -f $out/$r.ncu-rep
done
for c in C2 C4 C5; do timeout 300 python tools/timeline.py $c > $out/timeline_$c.txt 2>&1; done
for c in C1 C2 C3 C4 C5; do cut -c1-200 $out/bench_$c.jsonl; done; cut -c1-200 $out/bench_C2_ref.jsonl
