#!/bin/bash
out=gpurun_out/r02t; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python tools/sweep.py --configs C1,C2,C2,C3 --reps 7 --variants default,lloyd1 > $out/sweep.jsonl 2>&1; python tools/show_sweep.py $out/sweep.jsonl
