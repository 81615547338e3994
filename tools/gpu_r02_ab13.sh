# round-2 A/B 13: hub chunk / hub degree with the one-ahead claim
set -x
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C2 cc 9
