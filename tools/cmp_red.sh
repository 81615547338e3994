#!/bin/bash
# usage: tools/cmp_red.sh CONFIG ALG [sweep args] — sweep (adaptive tuned) with every exp_libs/*.so
cfg=$1; alg=$2; shift 2
for L in exp_libs/*.so; do
  AGRAPH_LIB=$PWD/$L timeout 300 python tools/sweep.py --config $cfg --sources 3 --reps 1 --alg $alg --orders 0 --only adaptive_tuned "$@" 2>&1 | grep -v config | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print('$L', d['alg'], round(d.get('ms_median',0),3), d.get('iters'), d.get('redundancy'), d.get('error',''))"
done
