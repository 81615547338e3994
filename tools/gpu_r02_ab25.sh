# round-2 A/B 25: unordered SSSP reads the expansion value L1-cacheable (stale-high is safe); acq_rel instead of SC fences in the grid barrier and hub drain
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size or c1_all or window or delta or no_parents or overflow or small_frontier or adaptive" > gpurun_out/pytest_ab25.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_ab25.log
timeout 1500 python -m pytest tests/test_gpu_static_full.py -x -q -m gpu --timeout 900 -k "unordered_sssp" > gpurun_out/pytest_ab25s.log 2>&1; echo "pytest static rc=$?"; tail -2 gpurun_out/pytest_ab25s.log
bash tools/cmp_libs.sh C2 sssp 25
bash tools/cmp_libs.sh C2 bfs 17
bash tools/cmp_libs.sh C4 sssp 5
bash tools/cmp_libs.sh C3 sssp 2
