python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "C4 or warp or wpq or shard or dense or auto or dist" > gpurun_out/d6_pytest.txt 2>&1; tail -2 gpurun_out/d6_pytest.txt
for v in 1 0; do echo "outlier tasks=$v"; SKNN_OUTLIER_TASKS=$v timeout 120 python tools/run_one.py C4 1.0 3; done
SKNN_OUTLIER_TASKS=0 SKNN_TILEPROF=1 timeout 120 python tools/run_one.py C4 1.0 1 2>&1 | grep tileprof | head -4
SKNN_TILEPROF=1 timeout 120 python tools/run_one.py C4 1.0 1 2>&1 | grep tileprof | head -4
timeout 300 python bench.py --config C4 --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | cut -c1-300
