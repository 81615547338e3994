#!/bin/bash
# usage: tools/cmp_sweep.sh OUTPREFIX CONFIG [sweep args...] — tools/sweep.py with every exp_libs/*.so
pre=$1; cfg=$2; shift 2
for L in exp_libs/*.so; do
  n=$(basename $L .so)
  AGRAPH_LIB=$PWD/$L timeout 600 python tools/sweep.py --config $cfg "$@" > gpurun_out/${pre}_${cfg}_${n}.jsonl 2>&1
done
