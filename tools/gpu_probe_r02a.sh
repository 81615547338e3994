# round-2 probe: random-gather throughput micro-benchmark + full ncu capture of C2 BFS/SSSP (reports kept)
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 ./tools/micro/gather_bench > gpurun_out/r02_gather_bench.txt 2>&1
cat gpurun_out/r02_gather_bench.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:traverse_kernel -s 2 -c 1 -o gpurun_out/r02a_bfs python tools/one_query.py --config C2 --alg bfs --n 3 > gpurun_out/ncu_bfs.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:traverse_kernel -s 2 -c 1 -o gpurun_out/r02a_sssp python tools/one_query.py --config C2 --alg sssp --n 3 > gpurun_out/ncu_sssp.log 2>&1
ls -la gpurun_out
