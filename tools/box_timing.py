#!/usr/bin/env python
"""Developer timing: flat BinMD vs MDBox BinMD (NEXT #4, extents computed once per event file)
on one config, CUDA events on the launching stream, mean of K calls.

  python tools/box_timing.py [--config corelli|topaz] [--nops N] [--box 32,256,1024]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="corelli")
    ap.add_argument("--nops", type=int, default=None)
    ap.add_argument("--box", default="32,256,1024")
    ap.add_argument("--iters", type=int, default=10)
    args = ap.parse_args()
    import torch
    import synth
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    wl = synth.make_workload(args.config, nops=args.nops)
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    ev = torch.from_numpy(synth.events_for_run(wl, 0, n=10_000_000)).cuda()

    def timed(fn):
        ts = []
        for it in range(args.iters + 2):
            m.mdnorm_reset(g)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            if it >= 2:
                ts.append(a.elapsed_time(b) * 1e3)
        return statistics.mean(ts), float(m.packed_histograms(g)[g.nbins_total:2 * g.nbins_total].sum().item())

    out = {"flat_us": timed(lambda: m.binmd_accumulate(g, wl.UB, wl.ops, ev))}
    for be in [int(x) for x in args.box.split(",")]:
        bounds = m.binmd_box_bounds(g, ev, be)
        t_b = timed(lambda: m.binmd_box_bounds(g, ev, be, bounds=bounds))[0]
        out[f"boxes{be}_us"] = timed(lambda: m.binmd_accumulate_boxes(g, wl.UB, wl.ops, ev, be, bounds))
        out[f"bounds{be}_us"] = t_b
    print(json.dumps(out))


if __name__ == "__main__":
    main()
