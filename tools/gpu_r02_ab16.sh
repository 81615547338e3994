# round-2 A/B 16: control-block lines spread, hub-ring poll backoff, no mid-iteration L1 invalidation in the hub drain
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_cc.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size or c1_all or small_frontier or window or delta" > gpurun_out/pytest_ab16.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab16.log
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C2 cc 9
bash tools/cmp_libs.sh C4 sssp 5
bash tools/cmp_libs.sh C3 sssp 2
for L in ref base; do for a in bfs sssp; do echo "== $L $a"; AGRAPH_LIB=$PWD/exp_libs/$L.so python tools/level_roofline.py --config C2 --alg $a; done; done
