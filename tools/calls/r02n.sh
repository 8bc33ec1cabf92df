#!/bin/bash
out=gpurun_out/r02n; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C5 0.01 1 > $out/smoke.txt 2>&1 || { echo smoke failed; tail -5 $out/smoke.txt; exit 1; }
timeout 1500 python -m pytest tests -x -q -m gpu > $out/pytest.txt 2>&1; tail -3 $out/pytest.txt
for v in cur nominfirst; do
  if [ $v = cur ]; then L=; else L=ab/$v.so; fi
  SKNN_LIB=$L timeout 300 python tools/sweep.py --configs C2,C3,C5 --reps 7 --variants default > $out/ab_$v.jsonl 2>&1
  echo $v; python tools/show_sweep.py $out/ab_$v.jsonl
done
