# round-2 measurement: per-iteration CTA timing (diagnostic build), bench line, ncu launch list, full ncu of BFS + SSSP
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for a in bfs sssp; do AGRAPH_LIB=$PWD/exp_libs/prof.so timeout 300 python tools/prof_iters.py --config C2 --alg $a --src 1 > gpurun_out/prof_iters_$a.txt 2>&1; done
cat gpurun_out/prof_iters_*.txt
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err; echo "bench rc=$?"
cat gpurun_out/r02_bench.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/b_ncu.log 2>&1; echo "ncu list rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:traverse_kernel -s 2 -c 1 -o gpurun_out/r02c_bfs python tools/one_query.py --config C2 --alg bfs --n 3 > gpurun_out/ncu_bfs.log 2>&1; echo "ncu bfs rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:traverse_kernel -s 2 -c 1 -o gpurun_out/r02c_sssp python tools/one_query.py --config C2 --alg sssp --n 3 > gpurun_out/ncu_sssp.log 2>&1; echo "ncu sssp rc=$?"
