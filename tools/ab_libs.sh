set -u
L=variants/lib_base.so,variants/lib_new.so,variants/lib_new896.so,variants/lib_new1024_3d1024.so
python tools/time_kernels.py --config corelli --iters 10 --libs $L
python tools/time_kernels.py --config topaz --nops 8 --iters 5 --libs $L
python tools/time_kernels.py --config topaz --nops 48 --iters 3 --libs $L
