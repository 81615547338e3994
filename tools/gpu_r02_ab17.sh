# round-2 A/B 17: deferred visited-bit merge for the general-kernel R-MAT BFS (with / without the extra barrier)
set -x
bash tools/cmp_libs.sh C2 bfs 17
for L in base novis1 spread; do echo "== $L bfs"; AGRAPH_LIB=$PWD/exp_libs/$L.so python tools/level_roofline.py --config C2 --alg bfs; done
