#!/bin/bash
# usage: tools/cmp_libs.sh CONFIG ALG ARGS...  — one_query with every exp_libs/*.so
cfg=$1; alg=$2; shift 2
for L in exp_libs/*.so; do
  echo "== $L"
  AGRAPH_LIB=$PWD/$L timeout 300 python tools/one_query.py --config $cfg --alg $alg --n 4 "$@" 2>&1 | tail -3
done
