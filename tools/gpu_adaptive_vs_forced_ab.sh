mkdir -p gpurun_out
{
for alg in bfs sssp; do
  for rep in 1 2; do
    printf "tuned          "; timeout 300 python tools/one_query.py --config C2 --alg $alg --n 17 --summary
    printf "nosmallhub     "; AG_SMALL_HUB_WS=0 timeout 300 python tools/one_query.py --config C2 --alg $alg --n 17 --summary
    printf "forcedH_paperk "; timeout 300 python tools/one_query.py --config C2 --alg $alg --n 17 --summary --mapping 4 --workset 2
  done
done
} 2>&1 | tee gpurun_out/r01_adaptive_vs_forcedH_ab.txt
