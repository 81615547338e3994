#!/bin/bash
# usage: tools/gpu_trace_ab.sh CONFIG ALGS "name:defs" ... — build one exp lib per spec on the box, then print
# the per-iteration trace (us) of the tuned adaptive policy with each (median of 2 sources x 3 reps)
cfg=$1; algs=$2; shift 2
mkdir -p exp_libs
for spec in "$@"; do
  name=${spec%%:*}; defs=${spec#*:}
  python -m paper_conf_ipps_lib13_b200.build --force $defs --out=exp_libs/$name.so > /dev/null 2>&1 || echo "build $name failed"
done
for alg in ${algs//,/ }; do
  for L in exp_libs/*.so; do
    AGRAPH_LIB=$PWD/$L timeout 300 python tools/sweep.py --config $cfg --sources 2 --reps 3 --alg $alg --orders 0 --only adaptive_tuned --trace 2>&1 | grep -v '"config"' | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print('$L'.split('/')[-1][:-3].ljust(10), d['alg'], round(d.get('ms_median',0),3), [t[3] for t in d.get('trace',[])][:18], d.get('error',''))"
  done
done
