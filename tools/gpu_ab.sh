#!/bin/bash
# usage: tools/gpu_ab.sh "name1:-DX=1 -DY=2" "name2:" ...  — build one exp lib per spec on the box, then
# compare them with one_query on C2 (bfs, sssp) and C4 (bfs, sssp).  Output under gpurun_out/ab_*.txt
mkdir -p exp_libs gpurun_out
for spec in "$@"; do
  name=${spec%%:*}; defs=${spec#*:}
  python -m paper_conf_ipps_lib13_b200.build --force $defs --out=exp_libs/$name.so > /dev/null 2>&1 || echo "build $name failed"
done
for cfg in ${AB_CONFIGS:-C2 C4}; do
  for alg in ${AB_ALGS:-bfs sssp}; do
    for L in exp_libs/*.so; do
      echo "== $cfg $alg $L"
      AGRAPH_LIB=$PWD/$L timeout 300 python tools/one_query.py --config $cfg --alg $alg --n ${AB_N:-6} --summary 2>&1 | tail -2
    done
  done
done
