#!/bin/bash
out=gpurun_out/r02s; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C4 0.01 1 mapping=thread > $out/smoke.txt 2>&1 || { echo smoke failed; tail -5 $out/smoke.txt; }
timeout 900 python tools/sweep.py --configs C3,C5 --reps 5 --variants default,walkassign > $out/sweep_assign.jsonl 2>&1; python tools/show_sweep.py $out/sweep_assign.jsonl
timeout 900 python tools/sweep.py --configs C4 --reps 3 --variants default,env:SKNN_TPQ_HIGHD=1+SKNN_X=1 > $out/sweep_c4.jsonl 2>&1; python tools/show_sweep.py $out/sweep_c4.jsonl
SKNN_TPQ_HIGHD=1 timeout 900 python tools/sweep.py --configs C4 --reps 3 --variants thread,sparse > $out/sweep_c4_tpq.jsonl 2>&1; python tools/show_sweep.py $out/sweep_c4_tpq.jsonl
