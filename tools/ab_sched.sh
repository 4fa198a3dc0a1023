#!/bin/bash
# A/B of the MDNorm schedules (fused vs split) on CORELLI and TOPAZ, then the GPU test suite.
#   gpurun -- 'bash tools/ab_sched.sh'
set -u
mkdir -p gpurun_out
for cfg in "corelli" "topaz --nops 8" "topaz --nops 48"; do
  for s in 0 2; do
    echo "== $cfg sched=$s"
    timeout 300 python tools/time_kernels.py --config $cfg --sched $s --iters 5 2>&1 | tail -1
  done
done
