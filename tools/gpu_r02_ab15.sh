# round-2 A/B 15: status reads from L2 (coherent with the relaxations' atomics) instead of L1-cacheable
set -x
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C4 sssp 5
bash tools/cmp_libs.sh C4 bfs 5
for L in ref bcg cg; do for a in bfs sssp; do echo "== $L $a"; AGRAPH_LIB=$PWD/exp_libs/$L.so python tools/level_roofline.py --config C2 --alg $a; done; done
