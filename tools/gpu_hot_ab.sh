#!/bin/bash
# Free-output BFS hot-target dedup A/B (AG_HOTBITS) + CC timings; output in gpurun_out/hot_ab.txt
mkdir -p exp_libs gpurun_out
for hb in 0 32768 131072; do
  python -m paper_conf_ipps_lib13_b200.build --force -DAG_HOTBITS=$hb --out=exp_libs/hot$hb.so > /dev/null 2>&1 || echo "build hot$hb failed"
done
{
for cfg in C2 C4; do
  for L in exp_libs/hot*.so; do
    echo "== $L"
    AGRAPH_LIB=$PWD/$L timeout 300 python tools/one_query.py --config $cfg --alg bfs --n 33 --summary
  done
  timeout 300 python tools/one_query.py --config $cfg --alg bfs --n 33 --summary --set free_ppm=0
  timeout 300 python tools/one_query.py --config $cfg --alg cc --n 6 --summary
  timeout 300 python tools/one_query.py --config $cfg --alg cc --n 6 --summary --set free_ppm=0
done
} 2>&1 | tee gpurun_out/hot_ab.txt
