#!/bin/bash
# L1/shared carveout + eager staging A/B: old staging (AG_WQ_EAGER=0) vs eager, driver default carveout vs
# auto-minimum; C2/C4 BFS + SSSP medians over 16 sources.  Output: gpurun_out/carve_ab.txt
mkdir -p exp_libs gpurun_out
python -m paper_conf_ipps_lib13_b200.build --force -DAG_WQ_EAGER=0 --out=exp_libs/wq0.so > /dev/null 2>&1 || echo "build failed"
{
for cfg in C2 C4; do
  for alg in bfs sssp; do
    echo "-- $cfg $alg: old staging, default carveout"
    AG_CARVEOUT=-1 AGRAPH_LIB=$PWD/exp_libs/wq0.so timeout 300 python tools/one_query.py --config $cfg --alg $alg --n 17 --summary
    echo "-- $cfg $alg: eager staging, default carveout"
    AG_CARVEOUT=-1 timeout 300 python tools/one_query.py --config $cfg --alg $alg --n 17 --summary
    echo "-- $cfg $alg: eager staging, auto carveout"
    timeout 300 python tools/one_query.py --config $cfg --alg $alg --n 17 --summary
  done
done
} 2>&1 | tee gpurun_out/carve_ab.txt
