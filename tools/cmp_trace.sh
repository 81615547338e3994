#!/bin/bash
# usage: tools/cmp_trace.sh CONFIG ALG — per-iteration trace (adaptive tuned) with every exp_libs/*.so
cfg=$1; alg=$2; shift 2
for L in exp_libs/*.so; do
  AGRAPH_LIB=$PWD/$L timeout 300 python tools/sweep.py --config $cfg --sources 2 --reps 2 --alg $alg --orders 0 --only adaptive_tuned --trace "$@" 2>&1 | grep -v config | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print('$L'.split('/')[-1], d['alg'], round(d.get('ms_median',0),3), d.get('redundancy'), [t[3] for t in d.get('trace',[])][:8], d.get('error',''))"
done
