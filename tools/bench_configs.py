#!/usr/bin/env python
"""Per-config throughput of the hot path on one GPU (all BASELINE.json configs), for DESIGN.md.

  python tools/bench_configs.py [--out profiles/r01_configs.md]

MDNorm pixel-trajectories/s and BinMD events/s, each kernel group timed alone with CUDA events
(mean of 3 after 1 warm-up), plus segments/s and (event, op) pairs/s.  The multi-run config is the
rotation scan of BASELINE configs[3] on ONE GPU (its 8-GPU form shards these runs); the stress
config uses a 10^8-event slice of its 10^9 events (host generation of 10^9 events is too slow).
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_sc_hahnfgmmshvvs24_b200 as m  # noqa: E402

CASES = [
    ("tiny", dict(), 1),
    ("corelli", dict(), 1),
    ("topaz", dict(nops=1), 1),
    ("topaz", dict(nops=8), 1),
    ("topaz", dict(nops=48), 1),
    ("multirun", dict(nruns=120, events_per_run=2_000_000), 120),
    ("stress", dict(events_per_run=100_000_000), 1),
    # coarse grids that fit shared memory: the privatised path (auto selection), and the same
    # grid forced onto global red.add for comparison
    ("corelli", dict(), 1, dict(nbins=(60, 60, 1), priv=-1)),
    ("corelli", dict(), 1, dict(nbins=(60, 60, 1), priv=0)),
    ("topaz", dict(nops=8, events_per_run=20_000_000), 1, dict(nbins=(20, 20, 20), priv=-1)),
    ("topaz", dict(nops=8, events_per_run=20_000_000), 1, dict(nbins=(20, 20, 20), priv=0)),
]


def timed(fn, iters=3):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(iters):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return float(np.mean(ts))


def run_case(name, kw, nruns_used, over=None):
    over = over or {}
    wl = synth.make_workload(name, **kw)
    if "nbins" in over:
        wl.nbins = np.array(over["nbins"], dtype=np.int64)
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    m.mdnorm_set_privatization(g, over.get("priv", -1))
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    t0 = time.time()
    ev = torch.from_numpy(synth.events_for_run(wl, 0)).cuda()
    gen_s = time.time() - t0
    R, c = wl.R[:nruns_used], wl.charge[:nruns_used]
    md = timed(lambda: m.mdnorm_accumulate_runs(g, wl.UB, R, c, wl.ops, wl.k_min, wl.k_max), iters=2 if nruns_used > 1 else 3)
    bm = timed(lambda: m.binmd_accumulate(g, wl.UB, wl.ops, ev))
    m.mdnorm_reset(g)
    m.mdnorm_stats(g, 1, read=False)
    m.mdnorm_accumulate_runs(g, wl.UB, R, c, wl.ops, wl.k_min, wl.k_max)
    m.binmd_accumulate(g, wl.UB, wl.ops, ev)
    st = m.mdnorm_stats(g, 0)
    traj = wl.npix * wl.nops * nruns_used
    row = {
        "config": name, "args": kw, "pixels": wl.npix, "ops": wl.nops, "runs": nruns_used,
        "grid": [int(x) for x in wl.nbins], "events": int(ev.shape[0]),
        "mdnorm_ms": md, "traj_per_s": traj / (md / 1e3), "hit_frac": st["hit_trajectories"] / traj,
        "segments": st["segments"], "segments_per_s": st["segments"] / (md / 1e3),
        "binmd_ms": bm, "events_per_s": ev.shape[0] / (bm / 1e3),
        "pairs_per_s": ev.shape[0] * wl.nops / (bm / 1e3), "inside_frac": st["event_op_inside"] / max(st["event_op_pairs"], 1),
        "event_gen_s": gen_s, "paths": list(m.mdnorm_accumulation_paths(g)),
    }
    g.close()
    del ev
    torch.cuda.empty_cache()
    return row


def write_md(rows, path, roofs_path=os.path.join(ROOT, "profiles", "r01_roofs.json")):
    roofs = json.load(open(roofs_path)) if os.path.exists(roofs_path) else {}
    aps = roofs.get("atomics_per_s", {})
    l2 = max((v.get("red_f64_random", 0) for v in aps.values()), default=0)
    out = ["| config | traj | grid | paths (MDNorm, BinMD) | MDNorm ms | traj/s | hit % | segments | seg/s | "
           "% L2 atomic roof | events | BinMD ms | events/s | (event,op)/s | inside % |",
           "|" + "---|" * 15]
    for r in rows:
        name = r["config"] + (f" ({r['args']['nops']} ops)" if "nops" in r["args"] else "")
        if r["config"] == "multirun":
            name += f" ({r['runs']} runs)"
        grid = "x".join(str(x) for x in r["grid"])
        roof = f"{100 * r['segments_per_s'] / l2:.0f}%" if l2 and r["paths"][0] == "global" else "—"
        out.append(f"| {name} | {r['pixels'] * r['ops'] * r['runs']:.3g} | {grid} | {', '.join(r['paths'])} | "
                   f"{r['mdnorm_ms']:.3f} | {r['traj_per_s']:.3g} | {100 * r['hit_frac']:.1f} | {r['segments']:.3g} | "
                   f"{r['segments_per_s']:.3g} | {roof} | {r['events']:.3g} | {r['binmd_ms']:.3f} | "
                   f"{r['events_per_s']:.3g} | {r['pairs_per_s']:.3g} | {100 * r['inside_frac']:.1f} |")
    with open(path, "w") as f:
        f.write("\n".join(out) + "\n")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--md", default="", help="also write the markdown table here")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "configs.json"))
    ap.add_argument("--only", default="")
    a = ap.parse_args()
    rows = []
    for case in CASES:
        name, kw, nr = case[:3]
        if a.only and name not in a.only.split(","):
            continue
        r = run_case(name, kw, nr, case[3] if len(case) > 3 else None)
        print(json.dumps(r), flush=True)
        rows.append(r)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump({"gpu": torch.cuda.get_device_name(0), "rows": rows}, f, indent=1)
    if a.md:
        write_md(rows, a.md)


if __name__ == "__main__":
    main()
