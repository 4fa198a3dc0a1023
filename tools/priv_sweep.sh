set -x
T="python tools/time_kernels.py --iters 5"
for nb in 16x16x1 60x60x1 100x100x1 150x150x1; do
 for pv in 0 1; do for acc in 1 0; do $T --config corelli --nbins $nb --priv $pv --acc $acc; done; done
done
for nb in 16x16x16 20x20x20 25x25x25; do
 for pv in 0 1; do $T --config topaz --nops 8 --events 20000000 --nbins $nb --priv $pv; done
done
$T --config tiny --priv 0; $T --config tiny --priv 1
$T --config corelli ; $T --config topaz --nops 8 --events 20000000
