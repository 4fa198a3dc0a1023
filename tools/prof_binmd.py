#!/usr/bin/env python
"""BinMD alone on the CORELLI-shaped (or TOPAZ-shaped) config: CUDA-event times at several event
counts (the fixed per-launch cost is the intercept) -- and a short loop to run under ncu.

  python tools/prof_binmd.py [--config corelli] [--nops N] [--iters K] [--ncu]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="corelli")
    ap.add_argument("--nops", type=int, default=None)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--order", default="morton")
    ap.add_argument("--ncu", action="store_true", help="3 launches only (for ncu -k binmd_kernel)")
    ap.add_argument("--sizes", default="1024,151552,1000000,3000000,10000000")
    ap.add_argument("--boxes", type=int, default=0, help="also time binmd_accumulate_boxes with this box size")
    args = ap.parse_args()
    import numpy as np
    import torch
    import synth
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    from paper_conf_sc_hahnfgmmshvvs24_b200 import build
    build.build()
    wl = synth.make_workload(args.config, nops=args.nops, events_per_run=10_000_000)
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    ev = torch.from_numpy(synth.events_for_run(wl, 0, order=args.order)).cuda()
    if args.ncu:
        for _ in range(3):
            m.binmd_accumulate(g, wl.UB, wl.ops, ev)
        torch.cuda.synchronize()
        return
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    out = {}
    for n in [int(x) for x in args.sizes.split(",")]:
        sub = ev[:n]
        ts = []
        for it in range(args.iters + 3):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            m.binmd_accumulate(g, wl.UB, wl.ops, sub)
            b.record()
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(a.elapsed_time(b))
        out[n] = (float(np.median(ts)), float(np.min(ts)))
        print(json.dumps({"lib": os.path.basename(os.environ.get("MDN_LIB_PATH", "default")), "events": n, "median_ms": out[n][0], "min_ms": out[n][1],
                          "GB/s": 16 * n / out[n][0] / 1e6}), flush=True)
        if args.boxes:
            res = {}
            bounds = m.binmd_box_bounds(g, sub, args.boxes)
            for what in ("bounds", "boxes"):
                ts = []
                for it in range(args.iters + 3):
                    flush.zero_()
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record()
                    if what == "bounds":
                        m.binmd_box_bounds(g, sub, args.boxes, bounds)
                    else:
                        m.binmd_accumulate_boxes(g, wl.UB, wl.ops, sub, args.boxes, bounds)
                    b.record()
                    torch.cuda.synchronize()
                    if it >= 3:
                        ts.append(a.elapsed_time(b))
                res[what] = float(np.median(ts))
            print(json.dumps({"events": n, "box_events": args.boxes, "bounds_ms": res["bounds"],
                              "binmd_boxes_ms": res["boxes"]}), flush=True)


if __name__ == "__main__":
    main()
