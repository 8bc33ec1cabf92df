#!/bin/bash
# Paper-style studies on synthetic data (run under gpurun), JSON lines into gpurun_out/study/:
#   ksweep.jsonl    k in {1, 8, 20, 64, 512} x {full (auto at k<=128), partial} on C2 / C3 (Fig. 10, Table V)
#   ablation.jsonl  landmarks x0.5..x2 (Fig. 11), thread vs warp per query (Fig. 12 / Table IV),
#                   basic per-lane walk vs warp-union walk, Lloyd 0/1/2, seeding, on C1-C3 (+ C5 subset)
out=gpurun_out/study; mkdir -p $out
for k in 1 8 20 64 512; do
  timeout 900 python tools/sweep.py --configs C2,C3 --k $k --reps 3 --variants sparse,partial >> $out/ksweep.jsonl 2>> $out/err.txt
done
timeout 1200 python tools/sweep.py --configs C1,C2,C3 --reps 3 \
  --variants default,cl_half,cl_0.7,cl_1.4,cl_double,thread,warp,env:SKNN_WALK=lane,lloyd0,lloyd1,paperseed,sparse >> $out/ablation.jsonl 2>> $out/err.txt
timeout 900 python tools/sweep.py --configs C5 --reps 2 --variants default,cl_0.7,cl_1.4,env:SKNN_WALK=lane,lloyd1 >> $out/ablation.jsonl 2>> $out/err.txt
