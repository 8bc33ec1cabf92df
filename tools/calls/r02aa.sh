#!/bin/bash
out=gpurun_out/r02aa; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for v in cur ab4x4 u16ab1 minb4 cur; do
  if [ $v = cur ]; then L=; else L=ab/$v.so; fi
  SKNN_LIB=$L timeout 300 python tools/sweep.py --configs C2,C1 --reps 9 --variants default > $out/ab_$v.jsonl 2>&1
  echo $v; python tools/show_sweep.py $out/ab_$v.jsonl
done
