#!/bin/bash
out=gpurun_out/r02v; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C5 0.01 1 > $out/smoke.txt 2>&1 || { echo smoke failed; tail -5 $out/smoke.txt; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "integer_workloads or real_workloads or full_size or deterministic or seed or index or dense" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 900 python tools/sweep.py --configs C3,C4,C5 --reps 5 --variants default > $out/sweep.jsonl 2>&1; python tools/show_sweep.py $out/sweep.jsonl
