# round-2 A/B 9: exact free output for unordered SSSP on skewed graphs
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size_configs or c1_all or free_output or window" > gpurun_out/pytest_ab9.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab9.log
bash tools/cmp_libs.sh C2 sssp 17
bash tools/cmp_libs.sh C2 bfs 5
