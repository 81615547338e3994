# round-2 A/B 11: hub-task claim depth (1 vs 2 tasks claimed ahead) and 2048-entry small-working-set chunks
set -x
for a in bfs sssp cc; do bash tools/cmp_libs.sh C2 $a 17; done
AGRAPH_LIB=$PWD/exp_libs/ca1.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "hubs or full_size_configs" > gpurun_out/pytest_ab11.log 2>&1; echo "pytest ca1 rc=$?"; tail -2 gpurun_out/pytest_ab11.log
