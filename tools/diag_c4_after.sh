python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "C4 or warp or wpq or shard or dense or auto" > gpurun_out/d5_pytest.txt 2>&1; tail -3 gpurun_out/d5_pytest.txt
SKNN_TILEPROF=1 timeout 120 python tools/diag_c4_slice1.py 2 1 2>&1 | tail -6
timeout 120 python tools/diag_c4_slice1.py 8 1 n_clusters_q=3000
timeout 120 python tools/run_one.py C4 1.0 3
timeout 900 python tools/shard_balance.py --config C4 --P 2,8 > gpurun_out/d5_shard_c4.jsonl 2>&1; cut -c1-250 gpurun_out/d5_shard_c4.jsonl
