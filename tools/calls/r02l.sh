#!/bin/bash
out=gpurun_out/r02l; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C4 0.01 1 force_path=dense > $out/dense_smoke.txt 2>&1 || { echo dense smoke failed; tail -5 $out/dense_smoke.txt; exit 1; }
timeout 90 python tools/run_one.py C5 0.01 1 > $out/assign_smoke.txt 2>&1 || { echo assign smoke failed; tail -5 $out/assign_smoke.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "dense or auto_switch or global_ub or merge or index or integer_workloads or real_workloads or deterministic or full_size" > $out/pytest.txt 2>&1; tail -3 $out/pytest.txt
CS=/usr/local/cuda/bin/compute-sanitizer
for c in "c4_auto:C4 0.003 1" "c4_dense:C4 0.003 1 force_path=dense"; do n=${c%%:*}; a=${c#*:};
  timeout 900 $CS --tool racecheck --error-exitcode 7 python tools/run_one.py $a > $out/san_racecheck_$n.txt 2>&1; echo "racecheck $n rc=$? $(grep SUMMARY $out/san_racecheck_$n.txt)"; done
timeout 600 python tools/sweep.py --configs C3,C4,C5 --reps 5 --variants default > $out/sweep.jsonl 2>&1
python tools/show_sweep.py $out/sweep.jsonl
for c in C4 C5; do timeout 300 python tools/timeline.py $c 1.0 2 > $out/timeline_$c.txt 2>&1; grep assign_tc $out/timeline_$c.txt | head -8; done
timeout 300 python bench.py --config C5 --mode target --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > $out/bench_c5_target.jsonl 2>$out/bench_c5_target.err
timeout 300 python bench.py --config C5 --mode target --global-ub --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > $out/bench_c5_target_gub.jsonl 2>$out/bench_c5_target_gub.err
cut -c1-400 $out/bench_c5_target*.jsonl; tail -3 $out/bench_c5_target_gub.err
