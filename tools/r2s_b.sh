#!/bin/bash
out=gpurun_out/r02s_b; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.txt 2>&1 || { tail $out/build.txt; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q > $out/pytest_gpu.txt 2>&1; echo "pytest rc=$?"; tail -5 $out/pytest_gpu.txt
timeout 600 python tools/ooc_bench.py --config C5 --batch 500000 > $out/ooc_c5.jsonl 2>&1; cat $out/ooc_c5.jsonl | cut -c1-250
timeout 600 python tools/ooc_bench.py --config C2 --batch 100000 > $out/ooc_c2.jsonl 2>&1; cat $out/ooc_c2.jsonl | cut -c1-250
for c in C2 C3 C4; do timeout 900 python tools/shard_balance.py --config $c > $out/shard_$c.jsonl 2>&1; cut -c1-260 $out/shard_$c.jsonl; done
