#!/bin/bash
# free-output threshold A/B on the tuned adaptive policy: per-iteration traces for C2, C4 (bfs, sssp)
for cfg in ${CFGS:-C2 C4}; do
  for fp in 0 3906 ${EXTRA_FP:-}; do
    timeout 400 python tools/sweep.py --config $cfg --sources 2 --reps 3 --alg bfs,sssp --orders 0 --only adaptive_tuned --trace --set free_ppm=$fp 2>&1 | grep -v '"config"' | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print('$cfg free_ppm=$fp'.ljust(20), d['alg'], round(d.get('ms_median',0),3), d.get('redundancy'), [t[3] for t in d.get('trace',[])][:20], d.get('error',''))"
  done
done
