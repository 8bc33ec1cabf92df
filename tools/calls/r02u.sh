#!/bin/bash
out=gpurun_out/r02u; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "level1 or integer_workloads or real_workloads or c2 or sphere or tiny or duplicates" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 900 python tools/sweep.py --configs C2,C2,C5 --reps 7 --variants default > $out/sweep.jsonl 2>&1; python tools/show_sweep.py $out/sweep.jsonl
timeout 300 python tools/timeline.py C2 1.0 2 > $out/timeline_C2.txt 2>&1; sort -k2 -n -r $out/timeline_C2.txt | head -8
