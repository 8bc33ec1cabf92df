#!/bin/bash
out=gpurun_out/r02x; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C5 0.01 1 > $out/smoke.txt 2>&1 || { echo smoke failed; tail -5 $out/smoke.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "member_sort or integer_workloads or real_workloads or full_size or big_cluster or duplicates or tiny" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 900 python tools/sweep.py --configs C2,C2,C1 --reps 7 --variants default > $out/sweep.jsonl 2>&1; python tools/show_sweep.py $out/sweep.jsonl
timeout 300 python tools/timeline.py C2 1.0 2 > $out/timeline_C2.txt 2>&1; sort -k2 -n -r $out/timeline_C2.txt | head -8; tail -1 $out/timeline_C2.txt
