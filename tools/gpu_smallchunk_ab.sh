#!/bin/bash
# A/B of the small-working-set hub chunking threshold (AG_SMALLCHUNK_PER_CTA) on C2, medians of 16 sources.
mkdir -p gpurun_out
{
for alg in bfs sssp; do
  for rep in 1 2; do
    for v in 32 0 8; do
      printf "smallchunk=%-3s " $v; AG_SMALLCHUNK_PER_CTA=$v timeout 300 python tools/one_query.py --config C2 --alg $alg --n 17 --summary
    done
  done
done
} 2>&1 | tee gpurun_out/r01_smallchunk_ab.txt
