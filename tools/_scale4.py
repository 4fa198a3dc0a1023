import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np, synth, bench
import paper_conf_sc_hahnfgmmshvvs24_b200 as m
wl = bench.make_bench_workload(1)
for rep in (1, 8):
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    m.mdnorm_set_instrument(g, np.tile(wl.pix_dir, (rep, 1)), np.tile(wl.solid, rep)); m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0)
    torch.cuda.synchronize()
    g.close()
