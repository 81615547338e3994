#!/bin/bash
# C2 BFS: which tuned-kernel feature costs against the forced-hybrid paper kernel (medians of 16 sources)
mkdir -p gpurun_out
{
for rep in 1 2; do
  printf "tuned           "; timeout 300 python tools/one_query.py --config C2 --alg bfs --n 17 --summary
  printf "tuned_nosmall   "; AG_SMALL_HUB_WS=0 AG_SMALLCHUNK_PER_CTA=0 timeout 300 python tools/one_query.py --config C2 --alg bfs --n 17 --summary
  printf "forcedH_paperk  "; timeout 300 python tools/one_query.py --config C2 --alg bfs --n 17 --summary --mapping 4 --workset 2
  printf "tuned_t_small0  "; AG_SMALL_WS=0 AG_SMALL_HUB_WS=0 timeout 300 python tools/one_query.py --config C2 --alg bfs --n 17 --summary
done
} 2>&1 | tee gpurun_out/r01_bfs_tuned_probe.txt
