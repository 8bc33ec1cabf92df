#!/bin/bash
# Quick GPU check used during development (under gpurun): focused parity
# tests, C4 stage times per path, the C2 live timeline, one bench line.
# Every step has its own short timeout (a hung kernel must not eat the call).
out=gpurun_out/${1:-chk}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
# hang guard: one small dense join first, 90 s
timeout 90 python tools/run_one.py C4 0.01 1 force_path=dense > $out/dense_smoke.txt 2>&1 || { echo "dense smoke failed rc=$?"; cat $out/dense_smoke.txt | tail -5; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "${TESTS:-dense or auto_switch or graph or merge or c1_bitexact or integer_workloads}" > $out/pytest.txt 2>&1
tail -3 $out/pytest.txt
for p in auto dense; do timeout 240 python tools/run_one.py C4 1.0 2 force_path=$p >> $out/c4.txt 2>&1; done
timeout 240 python tools/timeline.py C2 > $out/timeline_c2.txt 2>&1
timeout 300 python tools/merge_bench.py > $out/merge_bench.jsonl 2>&1
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $out/bench_c2.jsonl 2> $out/bench_c2.err
tail -3 $out/c4.txt; tail -2 $out/timeline_c2.txt; cat $out/merge_bench.jsonl; cut -c1-600 $out/bench_c2.jsonl
