# round-2 A/B 10: final pass as coalesced-read scatter to caller ids (degree layout) instead of a random gather
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_cc.py tests/test_dist.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size or c1_all or dist or no_parents or edge_cases or device_buffers" > gpurun_out/pytest_ab10.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab10.log
for a in bfs sssp cc; do bash tools/cmp_libs.sh C2 $a 17; done
