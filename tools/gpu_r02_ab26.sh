# round-2 A/B 26: BFS/CC hybrid mapping with 1 aligned piece per thread per step (default 2)
set -x
bash tools/cmp_libs.sh C2 bfs 25
bash tools/cmp_libs.sh C4 bfs 5
bash tools/cmp_libs.sh C2 cc 9
