# round-2 A/B 3: hybrid tile size cap; plus the dist (multi-GPU) tests after the streamed extraction
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_dist.py tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "dist or tiny_random or hubs_and_star or full_size_configs" > gpurun_out/pytest_ab3.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab3.log
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 17; done
for a in bfs sssp; do bash tools/cmp_libs.sh C4 $a 5; done
for a in bfs sssp; do bash tools/cmp_libs.sh C3 $a 3; done
