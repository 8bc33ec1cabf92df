#!/bin/bash
# GPU-box profiling pass for the round's evidence (run under gpurun):
#   tools/profile_round.sh <tag> [config]
# -> gpurun_out/prof_<tag>/: bench line (with cpu_baseline), reference-arm line,
#    ncu launch list of the same bench command, ncu --set full of the scan kernel.
tag=$1; cfg=${2:-C2}
out=gpurun_out/prof_$tag
mkdir -p $out
python -c "import __graft_entry__ as g; g.build()"
python bench.py --config $cfg > $out/bench_$cfg.jsonl 2> $out/bench_$cfg.err
python bench.py --config $cfg --impl reference --steps 2 --warmup 3 > $out/bench_${cfg}_ref.jsonl 2>> $out/bench_$cfg.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_$cfg.csv \
    python bench.py --config $cfg --steps 2 --warmup 3 --no-cpu-baseline > $out/ncu_launch_bench.txt 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_scan_tpq -c 1 -o $out/scan_$cfg \
    python bench.py --config $cfg --steps 1 --warmup 3 --no-cpu-baseline > $out/ncu_full.txt 2>&1
tail -1 $out/bench_$cfg.jsonl | cut -c1-300
