#!/bin/bash
out=gpurun_out/r02r; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C5 0.01 1 > $out/smoke.txt 2>&1 || { echo smoke failed; tail -5 $out/smoke.txt; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "integer_workloads or real_workloads or full_size or deterministic or c2 or graph" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 600 python tools/sweep.py --configs C2,C3,C5,C4 --reps 5 --variants default > $out/sweep.jsonl 2>&1; python tools/show_sweep.py $out/sweep.jsonl
for c in C5; do timeout 300 python tools/timeline.py $c 1.0 2 > $out/timeline_$c.txt 2>&1; grep assign_tc $out/timeline_$c.txt | head -8; done
