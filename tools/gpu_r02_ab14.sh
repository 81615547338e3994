# round-2 A/B 14: small-frontier mode threshold on hub graphs; unordered BFS on R-MAT in the tuned specialisation
set -x
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C2 cc 9
