python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for v in "2 1" "8 1 n_clusters_q=3000"; do
 echo "== $v default"; timeout 120 python tools/diag_c4_slice1.py $v
 echo "== $v thread/highd"; SKNN_TPQ_HIGHD=1 timeout 120 python tools/diag_c4_slice1.py $v mapping=1
 echo "== $v taskorder0"; SKNN_TASKORDER=0 timeout 120 python tools/diag_c4_slice1.py $v
 echo "== $v sparse only"; timeout 120 python tools/diag_c4_slice1.py $v force_path=1
 echo "== $v lloyd0"; timeout 120 python tools/diag_c4_slice1.py $v lloyd_iters=0
done
