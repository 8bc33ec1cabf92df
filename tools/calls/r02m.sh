#!/bin/bash
out=gpurun_out/r02m; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C5 0.01 1 > $out/smoke.txt 2>&1 || { echo smoke failed; tail -5 $out/smoke.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "integer_workloads or real_workloads or graph or dense or merge or index or global_ub or partial or large_k or batches" > $out/pytest.txt 2>&1; tail -3 $out/pytest.txt
timeout 600 python tools/sweep.py --configs C4,C5 --reps 5 --variants default > $out/sweep.jsonl 2>&1
python tools/show_sweep.py $out/sweep.jsonl
timeout 300 python tools/timeline.py C4 1.0 2 > $out/timeline_C4.txt 2>&1; tail -1 $out/timeline_C4.txt
