#!/bin/bash
out=gpurun_out/r02s_head; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.txt 2>&1 || { tail $out/build.txt; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q > $out/pytest_gpu.txt 2>&1; echo "pytest rc=$?"
tail -3 $out/pytest_gpu.txt
timeout 300 python bench.py --steps 10 --warmup 3 > $out/bench_c2.jsonl 2> $out/bench_c2.err
for c in C1 C3 C4 C5; do timeout 400 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline >> $out/bench_all.jsonl 2>> $out/bench_all.err; done
cut -c1-400 $out/bench_c2.jsonl; cut -c1-300 $out/bench_all.jsonl
