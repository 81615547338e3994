# round-2 A/B 22: general-kernel R-MAT BFS under the tuned decisions neither writes nor clears the unused update bitmap
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size_configs or c1_all or free_output or small_frontier" > gpurun_out/pytest_ab22.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_ab22.log
bash tools/cmp_libs.sh C2 bfs 25
