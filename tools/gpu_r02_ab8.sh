# round-2 A/B 8: L1 allocation only for the status of the hottest (highest-degree) ids of the degree layout
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_cc.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size_configs or c1_all" > gpurun_out/pytest_ab8.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab8.log
for a in sssp bfs cc; do bash tools/cmp_libs.sh C2 $a 17; done
