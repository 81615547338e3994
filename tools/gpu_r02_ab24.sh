# round-2 A/B 24: finer hub tasks for small working sets also in the general kernel (R-MAT BFS under the tuned policy)
set -x
AGRAPH_LIB=$PWD/exp_libs/scg1.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "hubs or full_size_configs or tiny_random" > gpurun_out/pytest_ab24.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_ab24.log
bash tools/cmp_libs.sh C2 bfs 25
for L in scg0 scg1; do echo "== $L"; AGRAPH_LIB=$PWD/exp_libs/$L.so python tools/level_roofline.py --config C2 --alg bfs | head -6; done
