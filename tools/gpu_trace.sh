python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in C2 C4 C3; do timeout 600 python tools/sweep.py --config $c --only adaptive_tuned --orders 0 --trace --sources 2 --reps 2 > gpurun_out/trace_$c.jsonl 2>&1; done
bash tools/cmp_libs.sh C2 bfs > gpurun_out/cmp_bfs.txt 2>&1
bash tools/cmp_libs.sh C2 sssp > gpurun_out/cmp_sssp.txt 2>&1
