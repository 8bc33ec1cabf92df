#!/bin/bash
out=gpurun_out/r02e; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
source tools/ncu_reduce.sh
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"^k_dense_exact" -c 1 -o $out/c4_dense_exact \
   python tools/run_one.py C4 1.0 1 > $out/ncu_dense.txt 2>&1
reduce $out/c4_dense_exact
timeout 600 python tools/sweep.py --configs C2,C3,C5 --reps 5 --variants default,env:SKNN_TOPK=heap4 > $out/sweep_heap4.jsonl 2>&1
timeout 900 python tools/sweep.py --configs C4 --reps 3 --variants default,tau25,tau50,tau75,dense > $out/sweep_c4.jsonl 2>&1
python tools/show_sweep.py $out/sweep_heap4.jsonl $out/sweep_c4.jsonl 2>/dev/null || cat $out/sweep_*.jsonl | cut -c1-300
