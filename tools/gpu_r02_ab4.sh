# round-2 A/B 4: distance-only SSSP state, row offsets without L1 allocation, SSSP at 6 CTAs/SM
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -m gpu --timeout 900 -k "tiny_random or window or delta or c1_all or hubs or full_size_configs or overflow or no_parents" --durations=15 > gpurun_out/pytest_ab4.log 2>&1; echo "pytest rc=$?"; tail -25 gpurun_out/pytest_ab4.log
for a in sssp bfs; do bash tools/cmp_libs.sh C2 $a 17; done
bash tools/cmp_libs.sh C4 sssp 5
bash tools/cmp_libs.sh C3 sssp 3
python tools/level_roofline.py --config C2 --alg bfs > gpurun_out/levels_C2_bfs.txt 2>&1
python tools/level_roofline.py --config C2 --alg sssp > gpurun_out/levels_C2_sssp.txt 2>&1
cat gpurun_out/levels_C2_*.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:traverse_kernel -s 2 -c 1 -o gpurun_out/r02b_sssp python tools/one_query.py --config C2 --alg sssp --n 3 > gpurun_out/ncu_sssp.log 2>&1; echo "ncu rc=$?"
