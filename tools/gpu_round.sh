#!/bin/bash
# One GPU session: smoke, GPU tests, bench, ncu launch list and a full capture of the hot
# kernels.  Logs land in gpurun_out/.  Usage (from this container):
#   gpurun --timeout 2400 -- 'bash tools/gpu_round.sh [quick]'
set -u
mkdir -p gpurun_out
OUT=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/gpu.txt 2>&1
MODE=${1:-full}  # quick | full | configs (full + the per-config table)
echo "== smoke" ; timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
echo "== pytest -m gpu"; timeout 1500 python -m pytest tests -m gpu -q -rf > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 $OUT/pytest_gpu.log
echo "== bench"; timeout 900 python bench.py --steps 10 --warmup 3 --json-out $OUT/bench.json > $OUT/bench.log 2>&1; echo "bench rc=$?"; tail -c 1500 $OUT/bench.log
if [ "$MODE" = "quick" ]; then exit 0; fi
echo "== ncu launch list"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_launch_bench.log 2>&1; echo "ncu list rc=$?"
echo "== ncu full (cull, walk, binmd, xs)"
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:'mdnorm_cull_kernel|mdnorm_walk_kernel|binmd_kernel|xs_kernel' -s 8 -c 4 \
  -o $OUT/prof_full -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
ls -la $OUT
if [ "$MODE" = "configs" ]; then
  echo "== per-config table"
  timeout 1500 python tools/bench_configs.py --md $OUT/configs.md > $OUT/configs.log 2>&1; echo "configs rc=$?"
fi
