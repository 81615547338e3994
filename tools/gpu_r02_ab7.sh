# round-2 A/B 7: SSSP tuning sweep for the distance-only state (pieces per thread, occupancy, tile and hub chunk)
set -x
for a in sssp; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C4 sssp 5
bash tools/cmp_libs.sh C2 bfs 9
bash tools/cmp_libs.sh C3 sssp 3
