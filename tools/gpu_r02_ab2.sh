# round-2 A/B 2: TMA bulk hub staging; adaptive-window controller variants
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
AGRAPH_LIB=$PWD/exp_libs/b_bulk.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 600 -k "tiny_random or c1_all or hubs_and_star or full_size_configs or small_frontier" 2>&1 | tail -1
for c in C2; do for a in bfs sssp; do bash tools/cmp_libs.sh $c $a 17; done; done
bash tools/cmp_libs.sh C4 sssp 5
for c in C3 C3p C4 C2; do bash tools/cmp_libs_set.sh $c sssp 4 --set sssp_window=4294967294; done
