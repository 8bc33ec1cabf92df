#!/bin/bash
out=gpurun_out/r02g; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "center_graph or c1_bitexact or real_workloads or deterministic or c2_full_size_graph" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 300 python tools/timeline.py C2 1.0 2 > $out/timeline_C2.txt 2>&1
timeout 300 python tools/sweep.py --configs C1,C2 --reps 7 --variants default,env:SKNN_LM_TILED=1,env:SKNN_CKNN_OLD=1 > $out/sweep.jsonl 2>&1
python tools/show_sweep.py $out/sweep.jsonl
sort -k2 -n -r $out/timeline_C2.txt | head -12; tail -1 $out/timeline_C2.txt
