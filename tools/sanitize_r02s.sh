#!/bin/bash
# compute-sanitizer over the kernels added in the second half of round 2:
# the thread-per-query partial merges (direct and cp.async-staged), the
# dense-only tiled kernel (low and high d), the basic KNN-TI arm, the balanced
# shard owner deal, the warp-per-query outlier tasks (C4 slice) and the
# out-of-core overlapped batches.   tools/sanitize_r02s.sh <tag>
# (Not run: compute-sanitizer was closed on the GPU pool late in round 2 --
# these kernels are covered by the bounds-checked parity tests instead.)
out=gpurun_out/${1:-san2}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
CS=/usr/local/cuda/bin/compute-sanitizer
run() {  # run <tool> <name> <args...>
  local tool=$1 name=$2; shift 2
  timeout 900 $CS --tool $tool --error-exitcode 7 --print-limit 20 python "$@" > $out/san_${tool}_$name.txt 2>&1
  echo "$tool $name rc=$? $(grep 'SUMMARY' $out/san_${tool}_$name.txt | tail -1)"
}
cat > /tmp/san_ooc.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch, datagen, paper_conf_icde_chends17_b200 as sknn
Q, T, k, _ = datagen.workload("C5", 0.002)
ix = sknn.build(torch.from_numpy(T).cuda())
pq = torch.from_numpy(Q).pin_memory()
oi = torch.empty((Q.shape[0], k), dtype=torch.int32).pin_memory()
od = torch.empty((Q.shape[0], k), dtype=torch.float32).pin_memory()
ix.query(pq, k, query_batch=1000, out=(oi, od))
ix.close()
print("ok")
PY
for tool in memcheck racecheck synccheck; do
  for form in direct staged warp; do
    SKNN_MERGE=$form run $tool merge_$form tools/merge_bench.py --nq 3000 --k 32 --P 3,8 --reps 1
  done
  run $tool brute_tiled tools/run_one.py C3 0.02 1 force_path=3
  run $tool dense_only_highd tools/run_one.py ARC 1.0 1
  run $tool basic tools/run_one.py C5 0.002 1 mapping=3
  run $tool shard_balanced tools/run_one.py C4 0.003 1 shard_count=3 shard_rank=1 shard_policy=1
  run $tool ooc_overlap /tmp/san_ooc.py
done
