#!/bin/bash
# Bench lines C1-C5 (C2 with the cpu_baseline) and the reference arm: tools/r2s_bench.sh <tag>
tag=${1:-bench}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.txt 2>&1 || { tail $out/build.txt; exit 1; }
timeout 600 python bench.py > $out/bench_C2.jsonl 2> $out/bench_C2.err
for c in C1 C3 C4 C5; do timeout 600 python bench.py --config $c --no-cpu-baseline > $out/bench_$c.jsonl 2> $out/bench_$c.err; done
timeout 900 python bench.py --impl reference > $out/bench_C2_ref.jsonl 2> $out/bench_C2_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_C2.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $out/ncu_launch.txt 2>&1
for c in C1 C2 C3 C4 C5; do cut -c1-180 $out/bench_$c.jsonl; done
