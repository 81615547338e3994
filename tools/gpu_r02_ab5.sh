# round-2 A/B 5: warp-task engine (warps claim 32 queue entries, drain hub tasks alone; no CTA barrier inside an iteration)
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "tiny_random or window or delta or c1_all or hubs or full_size_configs or overflow or no_parents or small_frontier or bitmap_tier" > gpurun_out/pytest_ab5.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab5.log
for L in exp_libs/bfst.so; do AGRAPH_LIB=$PWD/$L timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size_configs[C2]" > gpurun_out/pytest_ab5_bfst.log 2>&1; echo "pytest bfst rc=$?"; tail -2 gpurun_out/pytest_ab5_bfst.log; done
for a in sssp bfs; do bash tools/cmp_libs.sh C2 $a 17; done
for a in sssp bfs; do bash tools/cmp_libs.sh C4 $a 5; done
bash tools/cmp_libs.sh C3 sssp 3
