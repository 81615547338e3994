#!/bin/bash
# usage: tools/gpu_env_ab.sh "label:ENV=V ENV2=V2" "label2:" ...  — medians over 16 sources per env spec for
# AB_CONFIGS x AB_ALGS (default C2 C4 x bfs sssp).  Output: gpurun_out/env_ab.txt
mkdir -p gpurun_out
{
for cfg in ${AB_CONFIGS:-C2 C4}; do
  for alg in ${AB_ALGS:-bfs sssp}; do
    for spec in "$@"; do
      name=${spec%%:*}; envs=${spec#*:}
      printf "%-14s " "$name"
      env $envs timeout 300 python tools/one_query.py --config $cfg --alg $alg --n ${AB_N:-17} --summary $AB_EXTRA
    done
  done
done
} 2>&1 | tee gpurun_out/env_ab.txt
