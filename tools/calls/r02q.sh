#!/bin/bash
out=gpurun_out/r02q; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C5 0.01 1 > $out/smoke.txt 2>&1 || { echo smoke failed; tail -5 $out/smoke.txt; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "integer_workloads or real_workloads or full_size or deterministic" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
for v in cur ab16x2 ab16x4 ab4x2; do
  if [ $v = cur ]; then L=; else L=ab/$v.so; fi
  SKNN_LIB=$L timeout 300 python tools/sweep.py --configs C2,C3,C5 --reps 5 --variants default > $out/ab_$v.jsonl 2>&1
  echo $v; python tools/show_sweep.py $out/ab_$v.jsonl
done
timeout 300 python tools/sweep.py --configs C4 --reps 5 --variants default > $out/c4.jsonl 2>&1; python tools/show_sweep.py $out/c4.jsonl
for c in C4 C5; do timeout 300 python tools/timeline.py $c 1.0 2 > $out/timeline_$c.txt 2>&1; grep assign_tc $out/timeline_$c.txt | head -8; done
