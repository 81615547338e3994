# round-2 A/B 12: SSSP deferral windows on C2 with the distance-only state (runtime policy fields, one library)
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for hw in 1 2 3 4 8 16; do echo "hub_window=$hw"; timeout 300 python tools/one_query.py --config C2 --alg sssp --n 17 --summary --set sssp_hub_window=$hw 2>&1 | tail -1; done
for w in 10 25 50 100 200; do echo "window=$w"; timeout 300 python tools/one_query.py --config C2 --alg sssp --n 17 --summary --set sssp_window=$w 2>&1 | tail -1; done
for hw in 0 1 2 4; do echo "C4 hub_window=$hw"; timeout 300 python tools/one_query.py --config C4 --alg sssp --n 5 --summary --set sssp_hub_window=$hw 2>&1 | tail -1; done
