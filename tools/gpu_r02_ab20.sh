# round-2 A/B 20: BFS level array swizzled (32 x 32 transpose per 1024-id block) in the degree layout
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_dist.py -x -q -m gpu --timeout 900 -k "tiny_random or hubs or full_size_configs or c1_all or dist or edge_cases or device_buffers or no_parents" > gpurun_out/pytest_ab20.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_ab20.log
bash tools/cmp_libs.sh C2 bfs 25
for L in noswz swz; do echo "== $L bfs"; AGRAPH_LIB=$PWD/exp_libs/$L.so python tools/level_roofline.py --config C2 --alg bfs; done
