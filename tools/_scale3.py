import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np, synth, bench
import paper_conf_sc_hahnfgmmshvvs24_b200 as m
wl = bench.make_bench_workload(1)
for rep in (1, 2, 4, 8):
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    m.mdnorm_set_instrument(g, np.tile(wl.pix_dir, (rep, 1)), np.tile(wl.solid, rep)); m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    fn = lambda: m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0)
    fn(); torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    print("pixels x", rep, f"{min(ts):.3f} ms, {min(ts)/rep:.4f} ms per copy", flush=True)
    g.close()
