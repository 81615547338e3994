# per-CTA iteration timing with hub-task counts (diagnostic build)
set -x
for a in bfs sssp; do AGRAPH_LIB=$PWD/exp_libs/prof.so timeout 300 python tools/prof_iters.py --config C2 --alg $a --src 1 > gpurun_out/prof2_iters_$a.txt 2>&1; done
cat gpurun_out/prof2_iters_*.txt
