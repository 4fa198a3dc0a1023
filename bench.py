#!/usr/bin/env python
"""Benchmark of the MDNorm + BinMD cross-section hot path (BASELINE.json metric).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
  (N > 1: launched by torchrun, one process per GPU, NCCL)

Workload (BASELINE.json configs[1], the config the metric is quoted on):
CORELLI-shaped single run -- 372,736 pixels x 24 symmetry ops (6/mmm) = 8,945,664
pixel-trajectories, 600x600x1 HK0 grid, 10^7 events (70% diffuse, 30% Bragg, Morton order).
One step = mdnorm_reset + MDNorm + BinMD (+ one NCCL reduce of the packed [norm | binmd] buffer
when N > 1) + cross-section: Algorithm 1 for one file per GPU.  Weak scaling: rank r
processes run r of a rotation scan (omega = 17 + 3r degrees, its own seeded events), so per-GPU
work is fixed.  value = pixel-trajectories of all ranks / max-over-ranks step time.

Prints ONE JSON line on rank 0 (contract in the task statement; fields documented in DESIGN.md §6).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "MDNorm pixel-trajectories/s (full MDNorm+BinMD+xs step; BinMD events/s in 'secondary')"
UNIT = "pixel-trajectories/s"

# ----------------------------------------------------------------------------- roofline constants
# Algorithmic fp64 operations (IEEE +,-,*,/ each counted once) per unit.
OPS_PER_TRAJ = 24      # v = M q (9 mul + 6 add) + clip (3 x (1 div + 2 mul))
OPS_PER_HIT = 7        # F(k_in) interpolation (6) + Omega*c (1)
OPS_PER_SEG = 22       # crossing (3) + F(k2) (6) + midpoint (2) + 3 bin coords (9) + value (2)
OPS_PER_PAIR = 21      # x = N q (9 mul + 6 add) + 3 x (sub, mul)
BYTES_PER_EVENT = 16   # packed float4 (w, Qx, Qy, Qz), read once
FP64_LANES_PER_SM = 64  # B200 FP64 pipe: 64 DADD/DMUL/DFMA per SM per clock (37 TFLOP/s FMA-counted)


def fp64_peak_tops(sm_mhz: float, n_sm: int = 148) -> float:
    """Peak non-fused fp64 operations/s (T): the definition forbids FMA contraction, so every
    algorithmic + - * is one FP64-pipe instruction."""
    return n_sm * FP64_LANES_PER_SM * sm_mhz * 1e6 / 1e12


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f), "measured"
    return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


def ncu_traffic():
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f)
    return {}


def atomic_roof():
    """Measured fp64 red.global.add rate into an L2-resident histogram (tools/roofs.cu on a B200
    of this pool, committed as profiles/rNN_roofs.json; the newest file wins)."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*_roofs.json")))
    if not files:
        return None, None
    with open(files[-1]) as f:
        r = json.load(f)
    return float(r["atomics_per_s"]["corelli_600x600"]["red_f64_random"]), os.path.relpath(files[-1], ROOT)


# ----------------------------------------------------------------------------- clocks


class ClockSampler:
    """nvidia-smi-equivalent sampling (NVML) of SM clock and throttle reasons every ~5 ms (the
    timed region of a default run is only tens of milliseconds)."""

    def __init__(self, device_index: int):
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.names = {
                pynvml.nvmlClocksEventReasonGpuIdle: "gpu_idle",
                pynvml.nvmlClocksEventReasonApplicationsClocksSetting: "applications_clocks_setting",
                pynvml.nvmlClocksEventReasonSwPowerCap: "sw_power_cap",
                pynvml.nvmlClocksEventReasonHwSlowdown: "hw_slowdown",
                pynvml.nvmlClocksEventReasonSyncBoost: "sync_boost",
                pynvml.nvmlClocksEventReasonSwThermalSlowdown: "sw_thermal_slowdown",
                pynvml.nvmlClocksEventReasonHwThermalSlowdown: "hw_thermal_slowdown",
                pynvml.nvmlClocksEventReasonHwPowerBrakeSlowdown: "hw_power_brake_slowdown",
                pynvml.nvmlClocksEventReasonDisplayClockSetting: "display_clock_setting",
            }
        except Exception as e:  # pragma: no cover
            self.nv = None
            self.err = str(e)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.names.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            self._stop.wait(0.005)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.nv:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons - {"gpu_idle"}),
                "samples": len(self.samples)}


# ----------------------------------------------------------------------------- workload


def make_bench_workload(world: int):
    import synth
    wl = synth.make_workload("corelli")
    if world > 1:
        wl.R = np.stack([synth.rot_y(17.0 + 3.0 * r) for r in range(world)])
        wl.charge = np.ones(world)
    return wl


def config_dict(wl, world):
    return {"workload": "corelli (BASELINE.json configs[1])", "pixels": wl.npix, "ops": wl.nops,
            "runs_per_gpu": 1, "trajectories_per_gpu": wl.npix * wl.nops,
            "events_per_gpu": wl.events_per_run, "grid": [int(x) for x in wl.nbins],
            "grid_extent": [[float(a), float(b)] for a, b in zip(wl.lo, wl.hi)],
            "event_order": "coarse-Q Morton (MDBox/SaveMD order)", "acc": "fp64",
            "l2": "flushed between timed steps (256 MiB device write)",
            "parallelism": f"dp{world} (rank r = run r; one NCCL reduce of [norm|binmd])" if world > 1
            else "single GPU"}


# ----------------------------------------------------------------------------- reference arm


def run_reference(args, rank, world):
    """--impl reference: the fp64 CPU oracle as it stands, on this host, per-step bounded sample."""
    if rank != 0:
        return 0
    import oracle
    import synth
    oracle.build()
    wl = make_bench_workload(1)
    ev = synth.events_for_run(wl, 0)
    stride = args.ref_stride
    threads = host_threads()
    times = []
    for k in range(args.warmup + args.steps):
        t_md, t_bm, _, _ = oracle_timed(wl, ev, stride, threads)
        if k >= args.warmup:
            times.append(t_md + t_bm)
    traj = wl.npix * wl.nops / stride
    value = traj / statistics.mean(times)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * statistics.mean(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (seeded, SURVEY.md §8(d) recipe)", "config": config_dict(wl, 1),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": f"every {stride}th pixel (all 24 ops) and every {stride}th event "
                                       f"of the CORELLI-shaped run per step; the C oracle on {threads} host "
                                       f"threads ({host_cpu()}), private histograms per thread"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def host_cpu() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_timed(wl, ev, stride, threads):
    """The oracle as it stands on every stride-th pixel (all ops) and every stride-th event of run 0,
    on `threads` host threads: each thread calls the unchanged C oracle (ctypes releases the GIL)
    on an interleaved pixel shard and a contiguous event shard with its own histograms, summed in
    fixed order afterwards (S§8(d): "OpenMP over (r, s, pixel-chunk) and (s, event-chunk), with
    per-thread private fp64 histograms reduced in fixed thread order").  Returns (seconds of
    MDNorm, seconds of BinMD, norm, binmd)."""
    from concurrent.futures import ThreadPoolExecutor

    import oracle
    oracle.build()
    g = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R[:1], wl.UB, wl.ops, wl.W)
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    evs = np.ascontiguousarray(ev[::stride])
    cuts = np.linspace(0, len(evs), threads + 1).astype(np.int64)
    shards = [np.ascontiguousarray(evs[cuts[t]:cuts[t + 1]]) for t in range(threads)]

    def md(t):
        a = oracle.Accumulator(g.nbins)
        oracle.mdnorm(g, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, wl.charge[0], wl.k_min, wl.k_max,
                      pix_begin=t * stride, pix_stride=stride * threads, acc=a)
        return a

    def bm(t):
        a = oracle.Accumulator(g.nbins)
        oracle.binmd(g, N, shards[t], acc=a)
        return a

    with ThreadPoolExecutor(threads) as ex:
        t0 = time.perf_counter()
        na = list(ex.map(md, range(threads)))
        t1 = time.perf_counter()
        ba = list(ex.map(bm, range(threads)))
        t2 = time.perf_counter()
    norm = na[0].value()
    for a in na[1:]:
        norm = norm + a.value()
    bmh = ba[0].value()
    for a in ba[1:]:
        bmh = bmh + a.value()
    return t1 - t0, t2 - t1, norm, bmh


def host_threads() -> int:
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return max(1, os.cpu_count() or 1)


def cpu_baseline(wl, ev, stride):
    threads = host_threads()
    t_md, t_bm, _, _ = oracle_timed(wl, ev, stride, threads)
    secs = t_md + t_bm
    traj = wl.npix * wl.nops / stride
    # single-thread figure on an 8x smaller sample of the same run
    s1_md, s1_bm, _, _ = oracle_timed(wl, ev, 8 * stride, 1)
    return {"value": traj / secs, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"every {stride}th pixel (all {wl.nops} ops) + every {stride}th event of run 0 "
                      f"({traj:.0f} trajectories, {len(ev) // stride} events; "
                      f"MDNorm {t_md:.2f} s + BinMD {t_bm:.2f} s) on {threads} host threads "
                      f"({host_cpu()}), private histograms per thread",
            "events_per_s": (len(ev) / stride) / secs,
            "single_thread": {"value": (traj / 8) / (s1_md + s1_bm), "unit": UNIT,
                              "sample": f"every {8 * stride}th pixel and event, 1 thread"}}


# ----------------------------------------------------------------------------- our arm


def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    import synth
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    from paper_conf_sc_hahnfgmmshvvs24_b200 import build

    build.build()
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    wl = make_bench_workload(world)
    run = rank if world > 1 else 0
    ev = synth.events_for_run(wl, run)
    g = m.mdnorm_create_grid(local_rank, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    ev_dev = torch.from_numpy(ev).to(dev)
    packed = m.packed_histograms(g)
    xs_dev = torch.empty(g.nbins_total, dtype=torch.float64, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    R, c = wl.R[run], float(wl.charge[run])

    def step(ph):
        # ph: five phase events, or None (the headline pass: an event recorded between two
        # kernels costs a few microseconds of stream serialisation, ~4% of this step)
        rec = (lambda i: ph[i].record()) if ph is not None else (lambda i: None)
        m.mdnorm_reset(g)
        rec(0)
        m.mdnorm_accumulate(g, wl.UB, R, wl.ops, wl.k_min, wl.k_max, c)
        rec(1)
        m.binmd_accumulate(g, wl.UB, wl.ops, ev_dev)
        rec(2)
        if world > 1:
            m.reduce_packed(packed, dst=0)
        rec(3)
        if rank == 0:
            m.mdnorm_cross_section(g, xs_dev)
        rec(4)

    mk = lambda: [torch.cuda.Event(enable_timing=True) for _ in range(5)]  # noqa: E731
    # work counters from one untimed step (tracing; counted kernels are a separate variant)
    m.mdnorm_stats(g, 1, read=False)
    step(mk())
    stats = m.mdnorm_stats(g, 0)
    for _ in range(args.warmup):
        step(mk())
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    stops = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    phases = [mk() for _ in range(args.steps)]
    # Two timed passes of K steps each, both bracketed by barrier + synchronize: the headline pass
    # (step events only) gives `value`; the phase pass records an event between the kernels of
    # every step and gives the per-kernel times of the roofline.
    with ClockSampler(local_rank) as clk:
        for k in range(args.steps):
            flush.zero_()  # L2 flush (outside the timed events)
            starts[k].record()
            step(None)
            stops[k].record()
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    with ClockSampler(local_rank) as clk_ph:
        for k in range(args.steps):
            flush.zero_()
            step(phases[k])
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in zip(starts, stops)]
    total_ms = torch.tensor([sum(step_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(total_ms, op=dist.ReduceOp.MAX)
    total_ms = float(total_ms.item())
    ph_ms = {name: statistics.mean(p[i].elapsed_time(p[i + 1]) for p in phases)
             for i, name in enumerate(["mdnorm", "binmd", "reduce", "xs"])}

    # ---------------- end to end through the C ABI with HOST buffers (pinned), copies inside
    ev_pin = torch.from_numpy(ev).pin_memory()
    xs_pin = torch.empty(g.nbins_total, dtype=torch.float64).pin_memory()

    def step_e2e():
        m.mdnorm_reset(g)
        m.mdnorm_accumulate(g, wl.UB, R, wl.ops, wl.k_min, wl.k_max, c)
        m.binmd_accumulate(g, wl.UB, wl.ops, ev_pin)          # chunked H2D overlapped with scatter
        if world > 1:
            m.reduce_packed(packed, dst=0)
        if rank == 0:
            m.mdnorm_cross_section(g, xs_pin)                   # D2H + synchronise

    for _ in range(2):
        step_e2e()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e_starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    e_stops = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    with ClockSampler(local_rank) as clk_e2e:
        for k in range(args.steps):
            flush.zero_()
            e_starts[k].record()
            step_e2e()
            e_stops[k].record()
        torch.cuda.synchronize()
    e2e_ms = torch.tensor([sum(a.elapsed_time(b) for a, b in zip(e_starts, e_stops))], dtype=torch.float64,
                          device=dev)
    if world > 1:
        dist.all_reduce(e2e_ms, op=dist.ReduceOp.MAX)
    e2e_ms = float(e2e_ms.item())

    # sanity: the result of the last step is a real cross-section
    if rank == 0:
        xs_np = xs_pin.numpy()
        finite = np.isfinite(xs_np)
        assert finite.sum() > 1000, "cross-section has too few finite bins"

    traj_total = wl.npix * wl.nops * world
    ev_total = len(ev) * world
    ms_per_step = total_ms / args.steps
    value = traj_total / (ms_per_step / 1e3)

    peaks, peaks_src = measured_peaks()
    clocks = clk.summary()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    fp64_peak = fp64_peak_tops(sm_max)
    hbm = float(peaks["hbm_gbs"])
    traffic = ncu_traffic()
    kernels = {}
    md_ops = OPS_PER_TRAJ * stats["trajectories"] + OPS_PER_HIT * stats["hit_trajectories"] + \
        OPS_PER_SEG * stats["segments"]
    t = ph_ms["mdnorm"] / 1e3
    md_traffic = None
    if "mdnorm_cull_kernel" in traffic and "mdnorm_walk_kernel" in traffic:
        md_traffic = traffic["mdnorm_cull_kernel"] + traffic["mdnorm_walk_kernel"]
    alu = {"bound": "alu", "achieved": md_ops / t / 1e12, "peak": fp64_peak, "unit": "TFLOP/s",
           "frac": md_ops / t / 1e12 / fp64_peak,
           "peak_note": f"fp64 non-fused ops at {sm_max:.0f} MHz (148 SM x 64 lanes), DESIGN.md §4"}
    aroof, aroof_src = atomic_roof()
    if aroof:
        # one fp64 red.add per segment (M7): the tighter of the two roofs
        kernels["mdnorm"] = {"bound": "atomic", "achieved": stats["segments"] / t / 1e9, "peak": aroof / 1e9,
                             "unit": "Gatomic/s", "frac": stats["segments"] / t / aroof,
                             "peak_source": f"measured: {aroof_src} (fp64 red.global.add, L2-resident bins)",
                             "alu": alu}
    else:
        kernels["mdnorm"] = dict(alu, peak_source=f"{peaks_src}: MEASURED_PEAKS.json sm_max_mhz x 148 SM x 64 fp64 lanes")
    kernels["mdnorm"].update({"kernels": "mdnorm_cull_kernel + mdnorm_walk_kernel", "traffic": md_traffic,
                              "ms": ph_ms["mdnorm"], "ops_per_launch": md_ops,
                              "segments_per_launch": stats["segments"]})
    t = ph_ms["binmd"] / 1e3
    bm_bytes = BYTES_PER_EVENT * len(ev)
    kernels["binmd_kernel"] = {"bound": "hbm", "achieved": bm_bytes / t / 1e9, "peak": hbm,
                               "unit": "GB/s", "frac": bm_bytes / t / 1e9 / hbm,
                               "traffic": traffic.get("binmd_kernel"), "ms": ph_ms["binmd"],
                               "bytes_per_launch": bm_bytes}
    t = ph_ms["xs"] / 1e3
    if rank == 0 and t > 0:
        xs_bytes = 24 * g.nbins_total
        kernels["xs_kernel"] = {"bound": "hbm", "achieved": xs_bytes / t / 1e9, "peak": hbm, "unit": "GB/s",
                                "frac": xs_bytes / t / 1e9 / hbm, "ms": ph_ms["xs"]}
    dom = max(("mdnorm", "binmd_kernel"), key=lambda k: kernels[k]["ms"])
    roof = {k: kernels[dom][k] for k in ("bound", "achieved", "peak", "unit", "frac", "traffic")}
    roof["kernel"] = kernels[dom].get("kernels", dom)
    roof["peak_source"] = kernels[dom].get("peak_source", f"{peaks_src}: MEASURED_PEAKS.json hbm_gbs")

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded, SURVEY.md §8(d) CORELLI recipe)",
        "config": config_dict(wl, world),
        "secondary": {"binmd_events_per_s": ev_total / (ms_per_step / 1e3),
                      "mdnorm_kernel_traj_per_s": wl.npix * wl.nops / (ph_ms["mdnorm"] / 1e3),
                      "binmd_kernel_events_per_s": len(ev) / (ph_ms["binmd"] / 1e3),
                      "mdnorm_segments_per_s": stats["segments"] / (ph_ms["mdnorm"] / 1e3),
                      "phase_ms": ph_ms, "work_counts_rank0": stats,
                      "phase_pass": {"steps": args.steps, "clocks": clk_ph.summary(),
                                     "note": "per-kernel times (phase_ms, roofline) come from a second timed pass "
                                             "with an event between kernels; value comes from the pass without"}},
        "clocks": clocks,
        "e2e": {"value": traj_total / (e2e_ms / args.steps / 1e3), "unit": UNIT,
                "ms_per_step": e2e_ms / args.steps,
                "h2d_bytes_per_step": int(ev.nbytes) * world,
                "d2h_bytes_per_step": 8 * g.nbins_total,
                "clocks": clk_e2e.summary(),
                "path": "C ABI with pinned host events (chunked H2D overlapped with BinMD) and host xs"},
        "gpu_launches": args.steps * (3 + (1 if rank == 0 else 0)),  # cull, walk, binmd (+ xs)
        "roofline": roof,
        "kernels": kernels,
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(wl, ev, args.cpu_stride)
    if rank == 0:
        print(json.dumps(line), flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                json.dump(line, f, indent=1)
    g.close()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-stride", type=int, default=1, help="oracle sample: every n-th pixel and event")
    ap.add_argument("--ref-stride", type=int, default=1, help="--impl reference per-step sample stride")
    ap.add_argument("--json-out", default=None)
    ap.add_argument("--dist-backend", default="nccl",
                    help="nccl (production); gloo + MDN_BENCH_SHARED_GPU=1 exercises the N>1 code "
                         "path with every rank on GPU 0 (tests only; not a performance number)")
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("MDN_BENCH_SHARED_GPU") == "1":
        local_rank = 0
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            dist.init_process_group(args.dist_backend)
    try:
        return run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    sys.exit(main())
