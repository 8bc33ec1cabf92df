#!/bin/bash
out=gpurun_out/r02f; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "c1_bitexact or integer_workloads or index or seed or deterministic or real_workloads" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
for c in C2 C5 C4; do timeout 300 python tools/timeline.py $c 1.0 2 > $out/timeline_$c.txt 2>&1; done
timeout 600 python tools/sweep.py --configs C1,C2,C3,C5,C4 --reps 5 --variants default > $out/sweep.jsonl 2>&1
python tools/show_sweep.py $out/sweep.jsonl
