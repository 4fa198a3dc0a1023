#!/bin/bash
# One GPU session: smoke, GPU tests, bench (with the extra configs and the CPU baseline), the ncu
# launch list of the bench and a full capture of the hot kernels.  Logs land in gpurun_out/.
#   gpurun --timeout 2400 -- 'bash tools/gpu_round.sh [quick|full] [TAG]'
set -u
mkdir -p gpurun_out
OUT=gpurun_out
MODE=${1:-full}
TAG=${2:-r02}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/gpu.txt 2>&1
echo "== smoke" ; timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke.log
echo "== pytest -m gpu"; timeout 1500 python -m pytest tests -m gpu -q -rf > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.log
echo "== bench"; timeout 900 python bench.py --steps 20 --warmup 5 --json-out $OUT/bench.json > $OUT/bench.log 2>&1; echo "bench rc=$?"; tail -c 300 $OUT/bench.log
if [ "$MODE" = "quick" ]; then exit 0; fi
echo "== ncu launch list"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${TAG}_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --extra-configs "" > $OUT/ncu_launch_bench.log 2>&1; echo "ncu list rc=$?"
echo "== ncu full (cull, walk, binmd, plan, xs)"
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:'mdnorm_cull_kernel|mdnorm_walk_kernel|binmd_kernel|binmd_plan|xs_kernel' -s 10 -c 5 \
  -o $OUT/${TAG}_full -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline --extra-configs "" > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
ls -la $OUT
