#!/usr/bin/env python
"""Developer probe: BinMD and MDNorm of one CORELLI run issued back to back on one stream, or on
two streams at once (BinMD on a second stream), timed with CUDA events around both.

  python tools/concurrency_probe.py [--libs a.so,b.so] [--iters K] [--config corelli|topaz] [--nops N]
"""
import argparse
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(args):
    sys.path.insert(0, ROOT)
    import torch
    import synth
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    wl = synth.make_workload(args.config, nops=args.nops)
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    ev = torch.from_numpy(synth.events_for_run(wl, 0)).cuda()
    sa = torch.cuda.current_stream()
    sb = torch.cuda.Stream()
    out = {}
    for mode in ("serial", "concurrent"):
        ts = []
        for it in range(args.iters + 2):
            m.mdnorm_reset(g)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(sa)
            if mode == "serial":
                m.binmd_accumulate(g, wl.UB, wl.ops, ev, stream=sa)
                m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, stream=sa)
            else:
                sb.wait_stream(sa)
                m.binmd_accumulate(g, wl.UB, wl.ops, ev, stream=sb)
                m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, stream=sa)
                sa.wait_stream(sb)
            e1.record(sa)
            torch.cuda.synchronize()
            if it >= 2:
                ts.append(e0.elapsed_time(e1))
        out[mode] = statistics.mean(ts)
        out[mode + "_sum"] = float(m.packed_histograms(g)[: 2 * g.nbins_total].sum().item())
    print(json.dumps(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="corelli")
    ap.add_argument("--nops", type=int, default=None)
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--libs", default="")
    ap.add_argument("--child", action="store_true")
    args = ap.parse_args()
    if args.child:
        return child(args)
    for lib in [x for x in args.libs.split(",") if x] or [""]:
        env = dict(os.environ)
        if lib:
            env["MDN_LIB_PATH"] = os.path.abspath(lib)
        cmd = [sys.executable, __file__, "--child", "--config", args.config, "--iters", str(args.iters)]
        if args.nops:
            cmd += ["--nops", str(args.nops)]
        r = subprocess.run(cmd, env=env, capture_output=True, text=True)
        line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr[-500:]
        print(f"{os.path.basename(lib) or 'default'}: {line}", flush=True)


if __name__ == "__main__":
    main()
