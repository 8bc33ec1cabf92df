#!/bin/bash
# NEXT-3 under gpurun: tests of the basic KNN-TI arm, the three-arm study
# (tools/paper_study.py) and Table IV's warp efficiency of the level-2 scan
# kernels (basic vs Sweet) from ncu.   tools/paper_study_ncu.sh <tag>
out=gpurun_out/${1:-study}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.txt 2>&1 || { tail $out/build.txt; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q -k "merge or basic" > $out/pytest.txt 2>&1; tail -2 $out/pytest.txt
timeout 1500 python tools/paper_study.py ${STUDY_ARGS} > $out/study.jsonl 2> $out/study.err; tail -3 $out/study.err
cut -c1-250 $out/study.jsonl
M=smsp__thread_inst_executed_per_inst_executed.ratio,gpu__time_duration.sum,smsp__inst_executed.sum,dram__bytes_read.sum,lts__t_bytes.sum
for c in C1 C2 C3 C5; do
  sc=1.0; [ $c = C5 ] && sc=0.05
  for m in basic auto; do
    timeout 600 ncu --metrics $M --clock-control none -k regex:"k_scan_(basic|tpq|wpq)" --csv python tools/run_one.py $c $sc 1 mapping=$m > $out/warpeff_${c}_$m.csv 2> $out/warpeff_${c}_$m.err
  done
done
ls -la $out
