# round-2 A/B: warp-level dedup, adaptive order axis (NEXT-3); new parity tests; calibration X7/X8
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "adaptive_order or bitmap_tier" > gpurun_out/pytest_new.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_new.log
AGRAPH_LIB=$PWD/exp_libs/b_dedup.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 600 -k "tiny_random or c1_all or hubs_and_star or full_size_configs" 2>&1 | tail -1
for c in C2 C4; do for a in bfs sssp; do bash tools/cmp_libs.sh $c $a 9; done; done
for a in bfs sssp; do bash tools/cmp_libs.sh C3 $a 3; done
mkdir -p gpurun_out/r02_adapt
for c in C3 C3p C4 C2; do
  timeout 300 python tools/one_query.py --config $c --alg sssp --n 3 --summary 2>&1 | tail -1
  timeout 300 python tools/one_query.py --config $c --alg sssp --n 3 --summary --set sssp_window=4294967294 2>&1 | tail -1
  timeout 300 python tools/one_query.py --config $c --alg sssp --n 3 --summary --order 1 2>&1 | tail -1
  timeout 300 python tools/one_query.py --config $c --alg sssp --n 3 --summary --order 1 --delta 0 2>&1 | tail -1
done
