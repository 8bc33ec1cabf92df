import json, sys
for l in open(sys.argv[1]):
    if not l.startswith('{'):
        print(l.strip()[:200]); continue
    d = json.loads(l)
    print('%-6s %-11s ms=%8.3f min=%8.3f q/s=%.3g pruned=%.3f ev/q=%7.1f cand=%6.1f cev/q=%6.1f ins/q=%6.1f %s mq=%d map=%d L=%d' % (
        d['config'], d['variant'], d['ms_total'], d['ms_min'], d['queries_per_s'], d['pruned_pct'], d['evals_per_query'],
        d['cand_per_qcluster'], d['center_evals_per_query'], d.get('inserts_per_query', 0), d['stages'], d['mq'], d['mapping'], d['launches']))
