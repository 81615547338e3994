# round-2 A/B 18: reduction counters (it_edges, it_nv, free_any, pend_count, totals) on their own lines too
set -x
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C2 cc 9
bash tools/cmp_libs.sh C4 sssp 5
bash tools/cmp_libs.sh C4 bfs 5
bash tools/cmp_libs.sh C3 bfs 2
