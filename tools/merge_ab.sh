#!/bin/bash
# A/B of the partial-list merge forms at C5 target-sharded sizes (P = 2, 4, 8)
out=gpurun_out/${1:-merge_ab}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.txt 2>&1 || { tail $out/build.txt; exit 1; }
timeout 600 python -m pytest tests -m gpu -x -q -k "merge" > $out/pytest_merge.txt 2>&1; tail -2 $out/pytest_merge.txt
timeout 300 python tools/merge_bench.py --P 2,4,8 > $out/merge_tpq.jsonl 2>&1
SKNN_MERGE=warp timeout 300 python tools/merge_bench.py --P 2,4,8 > $out/merge_warp.jsonl 2>&1
timeout 300 python tools/merge_bench.py --P 8 --k 16 >> $out/merge_tpq.jsonl 2>&1
timeout 300 python tools/merge_bench.py --P 8 --k 20 >> $out/merge_tpq.jsonl 2>&1
SKNN_MERGE=warp timeout 300 python tools/merge_bench.py --P 8 --k 20 >> $out/merge_warp.jsonl 2>&1
cat $out/merge_tpq.jsonl $out/merge_warp.jsonl
if [ -n "$NCU" ]; then
  ncu --set full --import-source on --clock-control none -c 1 -k regex:"^k_merge" -o $out/merge_tpq_p8 python tools/merge_bench.py --reps 1 > $out/merge_ncu.txt 2>&1
  python profiles/ncu_summary.py $out/merge_tpq_p8.ncu-rep merge_tpq_p8 > $out/merge_tpq_p8.md 2>/dev/null
  python tools/ncu_lines.py $out/merge_tpq_p8.ncu-rep 40 > $out/merge_tpq_p8.lines.txt 2>/dev/null
  cat $out/merge_tpq_p8.md
fi
