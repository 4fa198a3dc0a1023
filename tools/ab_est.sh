#!/bin/bash
# A/B of two library variants on CORELLI, TOPAZ 48 ops, the multirun and CORELLI bench steps,
# then the GPU test suite on the in-tree library:  gpurun -- 'bash tools/ab_est.sh base new'
A=${1:-base}; B=${2:-new}
L=variants/lib_$A.so,variants/lib_$B.so
python tools/time_kernels.py --config corelli --iters 20 --libs $L
python tools/time_kernels.py --config corelli --iters 20 --libs $L
python tools/time_kernels.py --config topaz --nops 48 --iters 3 --libs $L
for lib in $A $B; do MDN_LIB_PATH=variants/lib_$lib.so python bench.py --config multirun --steps 3 --warmup 3 --extra-configs "" --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$lib multirun', d['ms_per_step'], d['secondary']['phase_ms'])"; done
for lib in $A $B; do MDN_LIB_PATH=variants/lib_$lib.so python bench.py --steps 10 --warmup 3 --extra-configs "" --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$lib corelli step', d['ms_per_step'], d['secondary']['phase_ms'])"; done
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
