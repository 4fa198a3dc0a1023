#!/bin/bash
# A/B of library variants (variants/lib_*.so, tools/variants.py) on CORELLI and TOPAZ
#   gpurun -- 'bash tools/ab_libs.sh lib_a.so,lib_b.so [corelli|all]'
set -u
L=$(echo "$1" | sed 's#\([^,]*\)#variants/\1#g')
python tools/time_kernels.py --config corelli --iters 10 --libs $L
python tools/time_kernels.py --config corelli --iters 10 --order shuffled --libs $L
if [ "${2:-all}" = "all" ]; then
python tools/time_kernels.py --config topaz --nops 8 --iters 5 --libs $L
python tools/time_kernels.py --config topaz --nops 48 --iters 3 --libs $L
fi
