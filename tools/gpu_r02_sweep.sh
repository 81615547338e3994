# round-2 static-vs-adaptive sweep (every run oracle-verified) + the paper's threshold calibration (X7, X8)
set -u
mkdir -p gpurun_out/sweeps
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for cfg in ${CONFIGS:-C2 C4 C3}; do
  timeout 600 python -m tests.oracle_expect --config $cfg --sources ${SOURCES:-2} --seed 3 -o /tmp/expect_$cfg.npz
  timeout "${PER_CONFIG_S:-900}" python tools/sweep.py --config "$cfg" --sources ${SOURCES:-2} --reps ${REPS:-2} --orders 0,1 --kinds 0,1 \
    --expect /tmp/expect_$cfg.npz > "gpurun_out/sweeps/r02_static_${cfg}.jsonl" 2> "gpurun_out/sweeps/r02_static_${cfg}.err"
  echo "$cfg rc=$?"
done
python tools/sweep_table.py gpurun_out/sweeps/r02_static_*.jsonl > gpurun_out/sweeps/r02_static_table.md
cat gpurun_out/sweeps/r02_static_table.md
for cfg in C2 C4; do timeout 600 python tools/calibrate.py --x7 --config $cfg --sources 1 --expect /tmp/expect_$cfg.npz > gpurun_out/sweeps/r02_x7_$cfg.jsonl 2>&1; echo "x7 $cfg rc=$?"; done
timeout 900 python tools/calibrate.py --x8 --config C4 --sources 2 --expect /tmp/expect_C4.npz > gpurun_out/sweeps/r02_x8_C4.jsonl 2>&1; echo "x8 rc=$?"
tail -20 gpurun_out/sweeps/r02_x8_C4.jsonl


du -sh gpurun_out gpurun_out/sweeps/*; rm -f gpurun_out/sweeps/*.err
