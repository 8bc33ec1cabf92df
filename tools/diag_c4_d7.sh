python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "C4 or warp or wpq or shard or dense or auto or dist" > gpurun_out/d7_pytest.txt 2>&1; tail -2 gpurun_out/d7_pytest.txt
for v in 1 0; do echo "outlier tasks=$v"; SKNN_OUTLIER_TASKS=$v timeout 120 python tools/run_one.py C4 1.0 3; done
bash tools/seed_ab.sh seed_ab1
