#!/bin/bash
out=gpurun_out/r02z; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "member_sort or center_graph or integer_workloads or real_workloads or big_cluster or duplicates or tiny or c2_full" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 900 python tools/sweep.py --configs C2,C2,C1,C3 --reps 7 --variants default > $out/sweep.jsonl 2>&1; python tools/show_sweep.py $out/sweep.jsonl
timeout 300 python tools/timeline.py C2 1.0 2 > $out/timeline_C2.txt 2>&1; sort -k2 -n -r $out/timeline_C2.txt | head -12; tail -1 $out/timeline_C2.txt
