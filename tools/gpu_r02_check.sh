# round-2 check: build, full GPU suite, C2/C3/C4 medians, short bench
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 2400 python -m pytest tests -x -q -m gpu --timeout 900 -k "${K:-not nothing}" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_gpu.log
for c in C2 C4; do for a in bfs sssp; do timeout 300 python tools/one_query.py --config $c --alg $a --n 9 --summary 2>&1 | tail -1; done; done
for a in bfs sssp; do timeout 300 python tools/one_query.py --config C3 --alg $a --n 3 --summary 2>&1 | tail -1; done
timeout 300 python tools/one_query.py --config C4 --alg sssp --n 3 --summary --order 1 2>&1 | tail -1
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err; echo "bench rc=$?"
cat gpurun_out/r02_bench.json
