# round-2 A/B 6: degree-binned working set (heavy elements expanded first, in small tiles)
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_cc.py -x -q -m gpu --timeout 900 -k "tiny_random or window or delta or c1_all or hubs or full_size or overflow or no_parents or small_frontier or bitmap_tier or free_output" > gpurun_out/pytest_ab6.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab6.log
AGRAPH_LIB=$PWD/exp_libs/bfst.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size_configs" > gpurun_out/pytest_ab6_bfst.log 2>&1; echo "pytest bfst rc=$?"; tail -2 gpurun_out/pytest_ab6_bfst.log
for a in sssp bfs cc; do bash tools/cmp_libs.sh C2 $a 17; done
python tools/level_roofline.py --config C2 --alg bfs > gpurun_out/levels_C2_bfs.txt 2>&1
python tools/level_roofline.py --config C2 --alg sssp > gpurun_out/levels_C2_sssp.txt 2>&1
cat gpurun_out/levels_C2_*.txt
