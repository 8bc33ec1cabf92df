#!/bin/bash
out=gpurun_out/r02i; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 python -m pytest tests -q -m gpu -x > $out/pytest_gpu.txt 2>&1; tail -3 $out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.txt 2>&1; tail -3 $out/smoke.txt
bash tools/sanitize.sh r02i > $out/sanitize_summary.txt 2>&1; cat $out/sanitize_summary.txt
