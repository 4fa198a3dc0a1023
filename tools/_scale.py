import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np, synth, bench
import paper_conf_sc_hahnfgmmshvvs24_b200 as m
wl = bench.make_bench_workload(1)
g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid); m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
mr = synth.make_workload("multirun", nruns=16)
for same in (True, False):
    for k in (1, 2, 4, 8, 16):
        R = np.stack([wl.R[0]] * k) if same else mr.R[:k]
        c = np.ones(k)
        fn = lambda: m.mdnorm_accumulate_runs(g, wl.UB, R, c, wl.ops, wl.k_min, wl.k_max)
        fn(); torch.cuda.synchronize()
        ts = []
        for _ in range(5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); fn(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
        print("same" if same else "scan", k, f"{min(ts):.3f} ms total, {min(ts)/k:.4f} ms per run", flush=True)
