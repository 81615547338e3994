# round-2 A/B 23: hub drain as 1 / 2 / 4 independent thread groups per CTA (named barriers)
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for L in g2 g4; do AGRAPH_LIB=$PWD/exp_libs/$L.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "hubs or full_size_configs or tiny_random" > gpurun_out/pytest_ab23_$L.log 2>&1; echo "pytest $L rc=$?"; tail -1 gpurun_out/pytest_ab23_$L.log; done
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 25; done
bash tools/cmp_libs.sh C2 cc 9
bash tools/cmp_libs.sh C4 sssp 5
