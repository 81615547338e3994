# round-2 A/B 19: hub drain stops claiming ahead when fewer than k x CTAs tasks are left (k = 0: always ahead)
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "hubs or full_size_configs or tiny_random" > gpurun_out/pytest_ab19.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_ab19.log
for a in bfs sssp; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C2 cc 9
