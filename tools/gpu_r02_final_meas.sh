# round-2 final measurement: ncu launch list of bench, full ncu captures of C2 BFS + SSSP, per-level tables,
# per-CTA iteration timing (diagnostic build exp_libs/prof.so)
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for a in bfs sssp; do timeout 300 python tools/level_roofline.py --config C2 --alg $a > gpurun_out/r02_levels_C2_$a.txt 2>&1; done
timeout 300 python tools/level_roofline.py --config C4 --alg bfs > gpurun_out/r02_levels_C4_bfs.txt 2>&1
timeout 300 python tools/level_roofline.py --config C4 --alg sssp > gpurun_out/r02_levels_C4_sssp.txt 2>&1
cat gpurun_out/r02_levels_*.txt
for a in bfs sssp; do AGRAPH_LIB=$PWD/exp_libs/prof.so timeout 300 python tools/prof_iters.py --config C2 --alg $a --src 1 > gpurun_out/r02_prof_iters_c2_$a.txt 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/b_ncu.log 2>&1; echo "ncu list rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:traverse_kernel -s 2 -c 1 -o gpurun_out/r02f_bfs python tools/one_query.py --config C2 --alg bfs --n 3 > gpurun_out/ncu_bfs.log 2>&1; echo "ncu bfs rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:traverse_kernel -s 2 -c 1 -o gpurun_out/r02f_sssp python tools/one_query.py --config C2 --alg sssp --n 3 > gpurun_out/ncu_sssp.log 2>&1; echo "ncu sssp rc=$?"
du -sh gpurun_out
