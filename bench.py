#!/usr/bin/env python
"""Benchmark of the MDNorm + BinMD cross-section hot path (BASELINE.json metric).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C]
  (N > 1: one process per GPU over NCCL -- under torchrun, or launched by bench.py itself)

Workload (BASELINE.json configs[1], the config the metric is quoted on):
CORELLI-shaped single run -- 372,736 pixels x 24 symmetry ops (6/mmm) = 8,945,664
pixel-trajectories, 600x600x1 HK0 grid, 10^7 events (70% diffuse, 30% Bragg, Morton order).
One step = mdnorm_reset + MDNorm + BinMD (+ one NCCL reduce of the packed [norm | binmd] buffer
when N > 1) + cross-section: Algorithm 1 for one file per GPU.  Weak scaling: rank r
processes run r of a rotation scan (omega = 17 + 3r degrees, its own seeded events), so per-GPU
work is fixed.  value = pixel-trajectories of all ranks / max-over-ranks step time.

The other BASELINE configs are timed in the same run (reported under "configs"; --config makes
one of them the headline): multirun = configs[3], the 120-run x 24-op scan strong-scaled over the
ranks; topaz = configs[2], 200^3 grid, 48 ops, 10^8 events (weak, N = 1 only by default); stress =
configs[4], 500^3 grid, 48 ops, 10^9 events for the job, strong-scaled with one reduce_scatter.

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


def ncu_binding():
    """Per-kernel utilisation of the resources that can bind it (tools/ncu_summarize.py from the
    committed ncu --set full capture)."""
    p = os.path.join(ROOT, "profiles", "ncu_binding.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f)
    return {"kernels": {}}


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
    c = r["atomics_per_s"]["corelli_600x600"]
    src = os.path.relpath(files[-1], ROOT)
    if "clock" in c:
        src += f" (SM {c['clock']['sm_mhz_median']} MHz median, throttle reasons {c['clock']['reasons']})"
    return float(c["red_f64_random"]), src


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
                             "cpu": host_cpu_info(),
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
    cpu = host_cpu_info()
    return {"value": traj / secs, "unit": UNIT, "cores": threads, "kind": "oracle",
            "cpu": cpu,
            "sample": f"every {stride}th pixel (all {wl.nops} ops) + every {stride}th event of run 0 "
                      f"({traj:.0f} trajectories, {len(ev) // stride} events; "
                      f"MDNorm {t_md:.2f} s + BinMD {t_bm:.2f} s) on {threads} host threads "
                      f"({host_cpu()}), private histograms per thread",
            "events_per_s": (len(ev) / stride) / secs,
            "single_thread": {"value": (traj / 8) / (s1_md + s1_bm), "unit": UNIT,
                              "sample": f"every {8 * stride}th pixel and event, 1 thread"}}


# ----------------------------------------------------------------------------- our arm


def host_cpu_info() -> dict:
    """CPU model, sockets, physical cores and the threads this process may use (S§8(d))."""
    info = {"model": host_cpu(), "threads_available": host_threads()}
    phys, sockets = set(), set()
    try:
        cur = {}
        for line in open("/proc/cpuinfo"):
            if not line.strip():
                if "physical id" in cur and "core id" in cur:
                    phys.add((cur["physical id"], cur["core id"]))
                    sockets.add(cur["physical id"])
                cur = {}
                continue
            k, _, v = line.partition(":")
            cur[k.strip()] = v.strip()
    except OSError:
        pass
    info["sockets"] = len(sockets) or None
    info["physical_cores"] = len(phys) or None
    return info


class Case:
    """One bench workload on this rank: its grid, its runs, its device events and the step."""

    def __init__(self, m, torch, synth, name, world, rank, local_rank, dev, nops=None):
        self.name, self.world, self.rank = name, world, rank
        if name == "corelli":
            # configs[1]; weak scaling: rank r processes run r of a rotation scan (omega = 17 + 3r)
            wl = synth.make_workload("corelli")
            if world > 1:
                wl.R = np.stack([synth.rot_y(17.0 + 3.0 * r) for r in range(world)])
                wl.charge = np.ones(world)
            self.runs = [rank if world > 1 else 0]
            self.scaling = "weak"
            ev = synth.events_for_run(wl, self.runs[0])
            self.ev_dev = torch.from_numpy(ev).to(dev)
            self.ev_host = ev
            self.event_note = "10^7 events per run (its own seeded draw, Morton order)"
        elif name == "multirun":
            # configs[3]: the 120-run x 24-op CORELLI scan strong-scaled over the ranks (contiguous
            # run blocks, Algorithm 1's range(rank, size)) with one collective
            wl = synth.make_workload("multirun")
            from paper_conf_sc_hahnfgmmshvvs24_b200 import plan_shards
            plan = plan_shards(world, rank, wl.nruns, wl.npix, wl.events_per_run)
            self.runs = plan.runs
            self.scaling = "strong"
            ev = synth.events_for_run(wl, self.runs[0])
            self.ev_dev = torch.from_numpy(ev).to(dev)
            self.ev_host = None
            self.event_note = ("10^7 events per run; each rank bins one seeded 10^7-event draw (its first "
                               "run's) once per run it owns (BinMD cost does not depend on the run index)")
        elif name == "topaz":
            # configs[2] at nops ops (default 48, m-3m); weak scaling like corelli
            wl = synth.make_workload("topaz", nops=nops or 48)
            if world > 1:
                wl.R = np.stack([synth.rot_y(33.0 + 3.0 * r) for r in range(world)])
                wl.charge = np.ones(world)
            self.runs = [rank if world > 1 else 0]
            self.scaling = "weak"
            ev = synth.events_for_run(wl, self.runs[0], n=10_000_000)
            ev_d = torch.from_numpy(ev).to(dev)
            self.ev_dev = torch.cat([ev_d] * 10)  # 10^8 events: ten copies of one Morton-ordered draw
            del ev_d
            self.ev_host = None
            self.event_note = "10^8 events per run = ten copies of one seeded Morton-ordered 10^7-event draw"
        elif name == "stress":
            # configs[4]: one TOPAZ-shaped run on the 500^3 grid (1 GB per histogram part: every
            # reduction goes to HBM), nops ops (default 48), 10^9 events for the whole job, strong-
            # scaled: pixels interleaved by rank, events in contiguous blocks, ONE reduce_scatter
            # (the grid is too large to gather) and a divide of each rank's bin block
            wl = synth.make_workload("stress", nops=nops or 48)
            from paper_conf_sc_hahnfgmmshvvs24_b200 import plan_shards
            total_ev = 1_000_000_000
            plan = plan_shards(world, rank, 1, wl.npix, total_ev)
            self.runs = [0]
            self.pix = (plan.pix_begin, plan.pix_stride)
            self.scaling = "strong"
            b, e = plan.event_ranges[0]
            ev = synth.events_for_run(wl, 0, n=10_000_000)
            ev_d = torch.from_numpy(ev).to(dev)
            self.ev_dev = torch.empty((e - b, 4), dtype=torch.float32, device=dev)
            for o in range(0, e - b, ev_d.shape[0]):  # copies of one Morton-ordered 10^7-event draw
                k = min(ev_d.shape[0], e - b - o)
                self.ev_dev[o:o + k] = ev_d[:k]
            del ev_d
            self.ev_host = None
            self.event_note = (f"10^9 events for the job ({e - b} on this rank) = copies of one seeded "
                               "Morton-ordered 10^7-event draw")
        else:
            raise ValueError(name)
        self.wl = wl
        self.m = m
        g = m.mdnorm_create_grid(local_rank, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
        m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
        m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
        self.g = g
        self.packed = m.packed_histograms(g)
        self.xs_dev = torch.empty(g.nbins_total, dtype=torch.float64, device=dev)
        self.traj_rank = len(self.runs) * wl.npix * wl.nops
        self.events_rank = len(self.runs) * self.ev_dev.shape[0]
        self.traj_total = (wl.nruns if name == "multirun" else world) * wl.npix * wl.nops
        self.events_total = self.events_rank * (1 if name == "multirun" else world) if name != "multirun" \
            else wl.nruns * self.ev_dev.shape[0]
        if name == "stress":
            pb, ps = self.pix
            self.traj_rank = len(range(pb, wl.npix, ps)) * wl.nops
            self.traj_total = wl.npix * wl.nops
            self.events_total = 1_000_000_000

    def step(self, ph=None, events=None):
        """mdnorm_reset + BinMD of this rank's runs' events + MDNorm of the runs (+ one reduce of
        [norm | binmd] when N > 1) + the cross-section on rank 0.  ph: five CUDA events recorded
        between the phases (the phase pass), or None (the headline pass)."""
        m, wl, g = self.m, self.wl, self.g
        rec = (lambda i: ph[i].record()) if ph is not None else (lambda i: None)
        m.mdnorm_reset(g)
        rec(0)

        def binmd():
            for _ in self.runs:
                m.binmd_accumulate(g, wl.UB, wl.ops, self.ev_dev if events is None else events)

        def mdnorm():
            if self.name == "stress":
                m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, float(wl.charge[0]),
                                    pix_begin=self.pix[0], pix_stride=self.pix[1])
            elif len(self.runs) == 1:
                r = self.runs[0]
                m.mdnorm_accumulate(g, wl.UB, wl.R[r], wl.ops, wl.k_min, wl.k_max, float(wl.charge[r]))
            else:
                m.mdnorm_accumulate_runs(g, wl.UB, wl.R[self.runs], wl.charge[self.runs], wl.ops, wl.k_min,
                                         wl.k_max)
        # Device events: BinMD first -- the MDNorm cull (programmatic dependent launch) takes the
        # SMs that BinMD's unevenly finishing CTAs leave.  Host events: MDNorm first, so that it
        # runs while the events are copied to the device.
        first, second = (binmd, mdnorm) if events is None else (mdnorm, binmd)
        first()
        rec(1)
        second()
        rec(2)
        if self.name == "stress" and self.world > 1:
            # the 2 GB [norm | binmd] is reduce-scattered; every rank divides its own bin block
            norm, bm, _ = m.reduce_scatter_packed(self.packed, nbins=g.nbins_total)
            rec(3)
            m.mdn_divide(norm, bm, xs=self.xs_dev[: norm.numel()])
            rec(4)
            return
        if self.world > 1:
            m.reduce_packed(self.packed, dst=0, nbins=g.nbins_total)
        rec(3)
        if self.rank == 0:
            m.mdnorm_cross_section(g, self.xs_dev if events is None else self.xs_out)
        rec(4)

    def config(self):
        wl = self.wl
        d = {"workload": {"corelli": "corelli (BASELINE.json configs[1])",
                          "multirun": "corelli multi-run rotation scan (BASELINE.json configs[3])",
                          "topaz": f"topaz, {wl.nops} ops (BASELINE.json configs[2])",
                          "stress": f"stress: 500^3 grid, {wl.nops} ops, 10^9 events (BASELINE.json configs[4])"
                          }[self.name],
             "pixels": wl.npix, "ops": wl.nops,
             "runs_total": wl.nruns if self.name == "multirun" else (1 if self.name == "stress" else self.world),
             "runs_per_gpu": len(self.runs), "trajectories_per_gpu": self.traj_rank,
             "events_per_gpu": self.events_rank, "events": self.event_note,
             "grid": [int(x) for x in wl.nbins],
             "grid_extent": [[float(a), float(b)] for a, b in zip(wl.lo, wl.hi)],
             "event_order": "coarse-Q Morton (MDBox/SaveMD order)", "acc": "fp64",
             "l2": "flushed between timed steps (256 MiB device write)"}
        if self.world > 1 and self.name == "stress":
            d["parallelism"] = (f"dp{self.world}: pixels interleaved by rank, events in contiguous blocks; "
                                "one NCCL reduce_scatter of [norm | binmd], each rank divides its bin block")
        elif self.world > 1:
            d["parallelism"] = (f"dp{self.world}: " + ("rank r = run r" if self.scaling == "weak"
                                                        else "contiguous run blocks per rank")
                                + "; one NCCL reduce of [norm | binmd] to rank 0")
        else:
            d["parallelism"] = "single GPU"
        return d


def time_case(case, args, steps, warmup, torch, dist, dev, flush, want_stats=True):
    """Warm-up, then a headline pass (step events only) and a phase pass (events between the
    kernels); both bracketed by barrier + synchronize; max over ranks of the summed step time."""
    m, world, local_rank = case.m, case.world, torch.cuda.current_device()
    mk = lambda: [torch.cuda.Event(enable_timing=True) for _ in range(5)]  # noqa: E731
    stats = None
    if want_stats:
        m.mdnorm_stats(case.g, 1, read=False)
        case.step(mk())
        stats = m.mdnorm_stats(case.g, 0)
    for _ in range(warmup):
        case.step(mk())
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    stops = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    phases = [mk() for _ in range(steps)]
    with ClockSampler(local_rank) as clk:
        for k in range(steps):
            flush.zero_()  # L2 flush (outside the timed events)
            starts[k].record()
            case.step(None)
            stops[k].record()
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    with ClockSampler(local_rank) as clk_ph:
        for k in range(steps):
            flush.zero_()
            case.step(phases[k])
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in zip(starts, stops)]
    total_ms = torch.tensor([sum(step_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(total_ms, op=dist.ReduceOp.MAX)
    total_ms = float(total_ms.item())
    # phase events in the device-event order (BinMD, then MDNorm)
    ph_ms = {name: statistics.mean(p[i].elapsed_time(p[i + 1]) for p in phases)
             for i, name in enumerate(["binmd", "mdnorm", "reduce", "xs"])}
    return {"ms_per_step": total_ms / steps, "phase_ms": ph_ms, "stats": stats, "clocks": clk.summary(),
            "clocks_phase": clk_ph.summary(), "step_ms_rank0": step_ms}


def case_summary(case, t, steps, warmup):
    ms = t["ms_per_step"]
    st = t["stats"] or {}
    out = {"metric": METRIC, "value": case.traj_total / (ms / 1e3), "unit": UNIT, "n_gpus": case.world,
           "steps": steps, "warmup": warmup, "ms_per_step": ms, "scaling": case.scaling,
           "config": case.config(), "clocks": t["clocks"],
           "binmd_events_per_s": case.events_total / (ms / 1e3),
           "phase_ms": t["phase_ms"],
           "mdnorm_kernel_traj_per_s": case.traj_rank / (t["phase_ms"]["mdnorm"] / 1e3),
           "binmd_kernel_events_per_s": case.events_rank / (t["phase_ms"]["binmd"] / 1e3),
           "work_counts_rank0": st}
    if st.get("segments"):
        out["mdnorm_segments_per_s"] = st["segments"] / (t["phase_ms"]["mdnorm"] / 1e3)
    return out


def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    import synth
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    from paper_conf_sc_hahnfgmmshvvs24_b200 import build

    build.build()
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    case = Case(m, torch, synth, args.config, world, rank, local_rank, dev, nops=args.nops)
    wl, g = case.wl, case.g
    t = time_case(case, args, args.steps, args.warmup, torch, dist, dev, flush)
    stats, ph_ms = t["stats"], t["phase_ms"]

    # ---------------- end to end through the C ABI with HOST buffers (pinned), copies inside
    e2e = None
    if case.ev_host is not None:
        ev_pin = torch.from_numpy(case.ev_host).pin_memory()
        xs_pin = torch.empty(g.nbins_total, dtype=torch.float64).pin_memory()
        case.xs_out = xs_pin
        for _ in range(2):
            case.step(None, events=ev_pin)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        e_starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
        e_stops = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
        with ClockSampler(local_rank) as clk_e2e:
            for k in range(args.steps):
                flush.zero_()
                e_starts[k].record()
                case.step(None, events=ev_pin)  # chunked H2D overlapped with BinMD; D2H xs + sync
                e_stops[k].record()
            torch.cuda.synchronize()
        e2e_ms = torch.tensor([sum(a.elapsed_time(b) for a, b in zip(e_starts, e_stops))], dtype=torch.float64,
                              device=dev)
        if world > 1:
            dist.all_reduce(e2e_ms, op=dist.ReduceOp.MAX)
        e2e_ms = float(e2e_ms.item())
        if rank == 0:
            assert np.isfinite(xs_pin.numpy()).sum() > 1000, "cross-section has too few finite bins"
        e2e = {"value": case.traj_total / (e2e_ms / args.steps / 1e3), "unit": UNIT,
               "ms_per_step": e2e_ms / args.steps,
               "h2d_bytes_per_step": int(case.ev_host.nbytes) * world,
               "d2h_bytes_per_step": 8 * g.nbins_total,
               "clocks": clk_e2e.summary(),
               "path": "C ABI with pinned host events (chunked H2D overlapped with BinMD) and host xs"}

    ms_per_step = t["ms_per_step"]
    value = case.traj_total / (ms_per_step / 1e3)
    peaks, peaks_src = measured_peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    fp64_peak = fp64_peak_tops(sm_max)
    hbm = float(peaks["hbm_gbs"])
    traffic = ncu_traffic()
    kernels = {}
    md_ops = OPS_PER_TRAJ * stats["trajectories"] + OPS_PER_HIT * stats["hit_trajectories"] + \
        OPS_PER_SEG * stats["segments"]
    tm = ph_ms["mdnorm"] / 1e3
    md_traffic = None
    if "mdnorm_cull_kernel" in traffic and "mdnorm_walk_kernel" in traffic:
        md_traffic = traffic["mdnorm_cull_kernel"] + traffic["mdnorm_walk_kernel"]
    alu = {"bound": "alu", "achieved": md_ops / tm / 1e12, "peak": fp64_peak, "unit": "TFLOP/s",
           "frac": md_ops / tm / 1e12 / fp64_peak,
           "peak_note": f"fp64 non-fused ops at {sm_max:.0f} MHz (148 SM x 64 lanes), DESIGN.md §4"}
    aroof, aroof_src = atomic_roof()
    if aroof:
        # one fp64 red.add per segment (M7): the tighter of the two roofs
        kernels["mdnorm"] = {"bound": "atomic", "achieved": stats["segments"] / tm / 1e9, "peak": aroof / 1e9,
                             "unit": "Gatomic/s", "frac": stats["segments"] / tm / aroof,
                             "peak_source": f"measured: {aroof_src} (fp64 red.global.add, L2-resident bins)",
                             "alu": alu}
    else:
        kernels["mdnorm"] = dict(alu, peak_source=f"{peaks_src}: MEASURED_PEAKS.json sm_max_mhz x 148 SM x 64 fp64 lanes")
    kernels["mdnorm"].update({"kernels": "mdnorm_cull_kernel + mdnorm_walk_kernel", "traffic": md_traffic,
                              "ms": ph_ms["mdnorm"], "ops_per_launch": md_ops,
                              "segments_per_launch": stats["segments"]})
    tb = ph_ms["binmd"] / 1e3
    bm_bytes = BYTES_PER_EVENT * case.events_rank
    kernels["binmd_kernel"] = {"bound": "hbm", "achieved": bm_bytes / tb / 1e9, "peak": hbm,
                               "unit": "GB/s", "frac": bm_bytes / tb / 1e9 / hbm,
                               "traffic": traffic.get("binmd_kernel"), "ms": ph_ms["binmd"],
                               "bytes_per_launch": bm_bytes,
                               "peak_source": f"{peaks_src}: MEASURED_PEAKS.json hbm_gbs"}
    if aroof:
        # the stream and the in-grid reductions do not overlap (profiles/r02_binmd_ablation.md):
        # serial floor = bytes at the measured copy bandwidth + reductions at the measured roof
        reds = stats["event_op_inside"]
        floor_s = bm_bytes / (hbm * 1e9) + reds / aroof
        kernels["binmd_kernel"]["serial_floor"] = {
            "bound": "hbm+atomic", "stream_us": bm_bytes / (hbm * 1e9) * 1e6, "reductions": reds,
            "reductions_us": reds / aroof * 1e6, "floor_us": floor_s * 1e6, "frac": floor_s / tb,
            "source": "profiles/r02_binmd_ablation.md (decisions hide under the stream; the reductions add to it)"}
    tx = ph_ms["xs"] / 1e3
    if rank == 0 and tx > 0:
        xs_bytes = 24 * g.nbins_total
        kernels["xs_kernel"] = {"bound": "hbm", "achieved": xs_bytes / tx / 1e9, "peak": hbm, "unit": "GB/s",
                                "frac": xs_bytes / tx / 1e9 / hbm, "ms": ph_ms["xs"]}
    nb = ncu_binding()
    walk = nb["kernels"].get("mdnorm_walk_kernel", {})
    if walk:
        kernels["mdnorm"]["binding"] = {
            "resource": "L1TEX data pipe: shared-memory flux look-ups + global fp64 reductions (walk)",
            "ncu_walk": walk, "ncu_cull": nb["kernels"].get("mdnorm_cull_kernel", {}), "source": nb.get("source")}
    if nb["kernels"].get("binmd_kernel"):
        kernels["binmd_kernel"]["binding"] = {
            "resource": "the event stream plus its in-grid fp64 L2 reductions, serialised (profiles/r02_binmd_ablation.md)",
            "ncu": nb["kernels"]["binmd_kernel"], "source": nb.get("source")}
    dom = max(("mdnorm", "binmd_kernel"), key=lambda k: kernels[k]["ms"])
    roof = {k: kernels[dom][k] for k in ("bound", "achieved", "peak", "unit", "frac", "traffic")}
    roof["kernel"] = kernels[dom].get("kernels", dom)
    roof["peak_source"] = kernels[dom].get("peak_source", f"{peaks_src}: MEASURED_PEAKS.json hbm_gbs")
    if "binding" in kernels[dom]:
        b = kernels[dom]["binding"]
        w = b.get("ncu_walk", b.get("ncu", {}))
        roof["binding_resource"] = {"resource": b["resource"],
                                    "l1tex_data_pipe_pct_of_peak": w.get("l1tex_data_pipe_pct"),
                                    "l2_red_sectors_pct_of_peak": w.get("l2_red_sectors_pct"),
                                    "source": b.get("source")}

    # our kernels per step: cull + walk per slab of every launch block (16 runs per block), one
    # binmd per run, the divide on rank 0
    blocks = -(-len(case.runs) // 16)
    slabs = m.mdnorm_debug_last_launch(case.g)["slabs"]
    launches_per_step = 2 * slabs * blocks + len(case.runs) + (1 if rank == 0 else 0)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": case.scaling,
        "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded, SURVEY.md §8(d) recipe)",
        "config": case.config(),
        "secondary": {"binmd_events_per_s": case.events_total / (ms_per_step / 1e3),
                      "mdnorm_kernel_traj_per_s": case.traj_rank / (ph_ms["mdnorm"] / 1e3),
                      "binmd_kernel_events_per_s": case.events_rank / (ph_ms["binmd"] / 1e3),
                      "mdnorm_segments_per_s": stats["segments"] / (ph_ms["mdnorm"] / 1e3),
                      "phase_ms": ph_ms, "work_counts_rank0": stats,
                      "phase_pass": {"steps": args.steps, "clocks": t["clocks_phase"],
                                     "note": "per-kernel times (phase_ms, roofline) come from a second timed pass "
                                             "with an event between kernels; value comes from the pass without"}},
        "clocks": t["clocks"],
        "gpu_launches": args.steps * launches_per_step,  # cull + walk per slab, binmd per run, xs on rank 0
        "roofline": roof,
        "kernels": kernels,
    }
    if e2e:
        line["e2e"] = e2e
    case.g.close()
    del case
    torch.cuda.empty_cache()
    # ---------------- the other BASELINE configs, measured in the same invocation
    extras = {}
    for name in [x for x in args.extra_configs.split(",") if x and x != args.config]:
        if name == "topaz" and world > 1 and not args.extra_weak:
            continue
        c2 = Case(m, torch, synth, name, world, rank, local_rank, dev, nops=None)
        steps2 = max(3, min(args.steps, 5))
        t2 = time_case(c2, args, steps2, 3, torch, dist, dev, flush)
        extras[name] = case_summary(c2, t2, steps2, 3)
        c2.g.close()
        del c2
        torch.cuda.empty_cache()
    if extras:
        line["configs"] = extras
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        wl0 = synth.make_workload("corelli")
        line["cpu_baseline"] = cpu_baseline(wl0, synth.events_for_run(wl0, 0), args.cpu_stride)
    if rank == 0:
        print(json.dumps(line), flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                json.dump(line, f, indent=1)
    return 0


def spawn_ranks(args) -> int:
    """`bench.py --gpus N` outside torchrun: launch N ranks with torch.distributed.run on
    127.0.0.1 (one process per GPU) and return their exit status."""
    import socket
    import subprocess
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.run(cmd).returncode


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", choices=["corelli", "multirun", "topaz", "stress"], default="corelli",
                    help="headline workload (default: BASELINE.json configs[1])")
    ap.add_argument("--nops", type=int, default=None, help="symmetry ops of the topaz / stress config (default 48)")
    ap.add_argument("--extra-configs", default="multirun,topaz,stress",
                    help="other BASELINE configs timed in the same run and reported under 'configs' ('' = none)")
    ap.add_argument("--extra-weak", action="store_true", help="also time the topaz extra at N > 1")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-stride", type=int, default=1, help="oracle sample: every n-th pixel and event")
    ap.add_argument("--ref-stride", type=int, default=1, help="--impl reference per-step sample stride")
    ap.add_argument("--json-out", default=None)
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        ap.error("at least 3 warm-up steps")
    world_env = os.environ.get("WORLD_SIZE")
    if world_env is None and args.gpus > 1:
        return spawn_ranks(args)
    world = int(world_env or "1")
    if world != args.gpus:
        ap.error(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    shared = os.environ.get("MDN_BENCH_SHARED_GPU") == "1"
    if shared:  # tests only: every rank on GPU 0 (NCCL refuses two ranks on one GPU: gloo)
        local_rank = 0
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        return run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    sys.exit(main())
