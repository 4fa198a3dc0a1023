import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np, synth, bench
import paper_conf_sc_hahnfgmmshvvs24_b200 as m
wl = bench.make_bench_workload(1)
g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid); m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
for k in (1, 8):
    R = np.stack([wl.R[0]] * k); c = np.ones(k)
    for _ in range(2):
        m.mdnorm_accumulate_runs(g, wl.UB, R, c, wl.ops, wl.k_min, wl.k_max)
    torch.cuda.synchronize()
