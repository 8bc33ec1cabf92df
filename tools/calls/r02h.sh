#!/bin/bash
out=gpurun_out/r02h; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 90 python tools/run_one.py C4 0.01 1 force_path=dense > $out/dense_smoke.txt 2>&1 || { echo dense smoke failed; tail -5 $out/dense_smoke.txt; exit 1; }
timeout 400 python -m pytest tests/test_gpu_parity.py -x -q -k "dense or auto_switch" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 300 python tools/sweep.py --configs C4 --reps 3 --variants default,tau50,dense > $out/sweep_c4.jsonl 2>&1
python tools/show_sweep.py $out/sweep_c4.jsonl
for v in cur u4 mb2 u4mb2; do
  if [ $v = cur ]; then L=; else L=ab/$v.so; fi
  SKNN_LIB=$L timeout 300 python tools/sweep.py --configs C5 --reps 3 --variants default > $out/c5_$v.jsonl 2>&1
  echo $v; python tools/show_sweep.py $out/c5_$v.jsonl
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"^k_dense_exact" -c 1 -o $out/c4_dense_exact \
   python tools/run_one.py C4 1.0 1 > $out/ncu_dense.txt 2>&1
source tools/ncu_reduce.sh; reduce $out/c4_dense_exact
tail -1 $out/c4_dense_exact.md | cut -d'|' -f2-20; head -12 $out/c4_dense_exact.lines.txt
