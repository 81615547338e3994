#!/bin/bash
# usage: tools/cmp_libs_set.sh CONFIG ALG N [one_query args...] — median device time with every exp_libs/*.so
cfg=$1; alg=$2; n=$3; shift 3
for L in exp_libs/*.so; do
  echo -n "$(basename $L) "
  AGRAPH_LIB=$PWD/$L timeout 600 python tools/one_query.py --config $cfg --alg $alg --n $n --summary "$@" 2>&1 | tail -1
done
