#!/bin/bash
# usage: tools/cmp_libs.sh CONFIG ALG [N] — median device time of N queries with every exp_libs/*.so
cfg=$1; alg=$2; n=${3:-9}
for L in exp_libs/*.so; do
  echo -n "$(basename $L) "
  AGRAPH_LIB=$PWD/$L timeout 300 python tools/one_query.py --config $cfg --alg $alg --n $n --summary 2>&1 | tail -1
done
