# round-2 full check: the whole GPU suite, bench line, per-config medians
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
timeout 2400 python -m pytest tests -x -q -m gpu --timeout 900 > gpurun_out/pytest_gpu_full.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu_full.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02_bench_full.json 2> gpurun_out/r02_bench_full.err; echo "bench rc=$?"
cat gpurun_out/r02_bench_full.json
