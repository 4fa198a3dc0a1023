#!/usr/bin/env python
"""Developer timing of the hot-path kernels on one config, for comparing build variants.

  python tools/time_kernels.py [--config corelli|topaz] [--nops N] [--iters K] [--libs a.so,b.so]

Each library is loaded in its own subprocess (MDN_LIB_PATH) and timed with CUDA events on the
launching stream: MDNorm (cull + walk) and BinMD separately, mean over K iterations after 2
warm-ups.  Prints one line per library.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(args):
    sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    import synth
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    wl = synth.make_workload(args.config, nops=args.nops,
                             events_per_run=args.events if args.events else None)
    nbins = [int(x) for x in args.nbins.split("x")] if args.nbins else wl.nbins
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, nbins, wl.W, args.acc)
    m.mdnorm_set_privatization(g, args.priv)
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    ev = torch.from_numpy(synth.events_for_run(wl, 0, order=args.order)).cuda()
    ts = {"mdnorm": [], "binmd": []}
    for it in range(args.iters + 2):
        m.mdnorm_reset(g)
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record()
        m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0)
        e[1].record()
        m.binmd_accumulate(g, wl.UB, wl.ops, ev)
        e[2].record()
        torch.cuda.synchronize()
        if it >= 2:
            ts["mdnorm"].append(e[0].elapsed_time(e[1]))
            ts["binmd"].append(e[1].elapsed_time(e[2]))
    m.mdnorm_stats(g, 1, read=False)
    m.mdnorm_reset(g)
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0)
    st = m.mdnorm_stats(g, 0)
    out = {k: float(np.mean(v)) for k, v in ts.items()}
    out["segments"] = st["segments"]
    out["paths"] = m.mdnorm_accumulation_paths(g)
    out["norm_sum"] = float(m.packed_histograms(g)[: g.nbins_total].sum().item())
    print(json.dumps(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="corelli")
    ap.add_argument("--nops", type=int, default=None)
    ap.add_argument("--events", type=int, default=0)
    ap.add_argument("--order", default="morton", help="event order: morton | shuffled")
    ap.add_argument("--iters", type=int, default=5)
    ap.add_argument("--libs", default="")
    ap.add_argument("--nbins", default="", help="override the grid, e.g. 60x60x1")
    ap.add_argument("--priv", type=int, default=-1, help="privatisation: -1 auto, 0 off, 1 on")
    ap.add_argument("--acc", type=int, default=1, help="1 = MDN_ACC_F64, 0 = MDN_ACC_F32")
    ap.add_argument("--child", action="store_true")
    args = ap.parse_args()
    if args.child:
        return child(args)
    libs = [x for x in args.libs.split(",") if x] or [""]
    for lib in libs:
        env = dict(os.environ)
        if lib:
            env["MDN_LIB_PATH"] = os.path.abspath(lib)
        cmd = [sys.executable, __file__, "--child", "--config", args.config, "--iters", str(args.iters),
               "--events", str(args.events), "--order", args.order, "--priv", str(args.priv),
               "--acc", str(args.acc)]
        if args.nbins:
            cmd += ["--nbins", args.nbins]
        if args.nops:
            cmd += ["--nops", str(args.nops)]
        r = subprocess.run(cmd, env=env, capture_output=True, text=True)
        line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr[-500:]
        print(f"{os.path.basename(lib) or 'default'}: {line}", flush=True)


if __name__ == "__main__":
    main()
