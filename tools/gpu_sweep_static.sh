#!/bin/bash
# Static variants (paper kernels and tuned kernels, both orders) vs the two adaptive policies on the
# single-GPU configs: the paper's Tables 2/3 study on B200.  Each config bounded by its own timeout;
# sweep.py flushes one JSON line per variant, so a timed-out config keeps its finished rows.
#   gpurun --timeout 2400 -- 'bash tools/gpu_sweep_static.sh'
set -u
mkdir -p gpurun_out/sweeps
for cfg in ${CONFIGS:-C2 C4 C3}; do
  timeout "${PER_CONFIG_S:-600}" python tools/sweep.py --config "$cfg" --sources ${SOURCES:-2} --reps ${REPS:-2} --orders 0,1 --kinds 0,1 \
    > "gpurun_out/sweeps/r01_static_${cfg}.jsonl" 2> "gpurun_out/sweeps/r01_static_${cfg}.err"
  echo "$cfg rc=$?"
done
python tools/sweep_table.py gpurun_out/sweeps/r01_static_*.jsonl > gpurun_out/sweeps/r01_static_table.md
cat gpurun_out/sweeps/r01_static_table.md
