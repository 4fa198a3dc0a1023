# ncu --set full with source of one config's MDNorm / BinMD kernels (tools/ncu_lines.py reads it)
#   gpurun -- 'bash tools/prof_src.sh TAG REGEX [time_kernels args...]'
set -u
OUT=gpurun_out
TAG=$1; RE=$2; shift 2
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$RE" -s 1 -c 1 -o $OUT/src_$TAG -f \
  python tools/time_kernels.py --child --iters 1 "$@" > $OUT/prof_$TAG.log 2>&1; echo "ncu rc=$?"
