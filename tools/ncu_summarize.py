#!/usr/bin/env python
"""Summarise ncu outputs from gpurun_out/ into profiles/ (tracked).

  python tools/ncu_summarize.py --tag r01 [--launches gpurun_out/launches.csv]
                                [--full gpurun_out/prof_full.ncu-rep]

Writes profiles/<tag>_launches.md (per-kernel device time and share of the bench step, from
the `--metrics gpu__time_duration.sum --clock-control none` launch list), profiles/
<tag>_ncu_full.md (key metrics of the `--set full` capture per kernel) and updates
profiles/ncu_traffic.json (DRAM bytes per launch, read by bench.py's roofline `traffic`).
"""
import argparse
import collections
import csv
import io
import json
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")
OURS = re.compile(r"(mdnorm_cull_kernel|mdnorm_walk_kernel|binmd_plan_kernel|binmd_kernel|xs_kernel|debug_\w+|pixels_prepare_kernel)")

KEY_METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
    "inst_executed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__thread_inst_executed_per_inst_executed.ratio", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "TPC.TriageCompute.sm__pipe_fp64_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sectors_srcunit_tex_op_red.sum", "lts__t_sectors_srcunit_tex_op_red.sum.pct_of_peak_sustained_elapsed",
    "lts__t_sectors.sum.pct_of_peak_sustained_elapsed", "launch__registers_per_thread", "launch__grid_size",
    "launch__block_size", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    # the L1TEX data pipe (shared-memory look-ups and global reductions share it: the walk's
    # binding resource), its shared-memory part, bank conflicts, global-reduction wavefronts
    "l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "l1tex__t_output_wavefronts_pipe_lsu_mem_global_op_red.sum.pct_of_peak_sustained_elapsed",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "sm__cycles_active.avg", "sm__cycles_active.max", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
]


def short(name):
    m = OURS.search(name)
    if m:
        t = re.match(r"<([^>]*)>", name[m.end():])
        return m.group(1) + (f"<{t.group(1)}>" if t else "")
    return name[:60]


def launches(path, tag):
    rows = list(csv.reader(open(path)))
    hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr_i]
    iK, iM, iV = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    tot = collections.Counter()
    cnt = collections.Counter()
    for r in rows[hdr_i + 1:]:
        if len(r) != len(h) or r[iM] != "gpu__time_duration.sum":
            continue
        v = float(r[iV].replace(",", ""))
        unit = r[h.index("Metric Unit")] if "Metric Unit" in h else "ns"
        v = v * {"ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(unit, 1e-3)
        k = short(r[iK])
        tot[k] += v
        cnt[k] += 1
    ours = {k: v for k, v in tot.items() if OURS.search(k)}
    step = sum(v for k, v in ours.items() if not k.startswith("debug") and "prepare" not in k)
    lines = [f"# {tag}: ncu launch list (gpu__time_duration.sum, --clock-control none)", "",
             "Cold-cache, serialised per-launch times of `python bench.py --steps 2 --warmup 3 "
             "--no-cpu-baseline` (all launches, incl. the stats/warm-up steps).  Compare SHARES, not "
             "absolutes.", "", "| kernel | launches | total us | mean us | share of our step kernels |",
             "|---|---|---|---|---|"]
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        share = f"{100 * v / step:.1f}%" if k in ours and step and "prepare" not in k else ""
        lines.append(f"| `{k}` | {cnt[k]} | {v:.1f} | {v / cnt[k]:.2f} | {share} |")
    with open(os.path.join(PROF, f"{tag}_launches.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))


def full(path, tag):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    data = rows[2:]
    traffic_p = os.path.join(PROF, "ncu_traffic.json")
    traffic = json.load(open(traffic_p)) if os.path.exists(traffic_p) else {}
    lines = [f"# {tag}: ncu --set full --clock-control none (one capture per kernel)", ""]
    per = collections.defaultdict(list)
    for r in data:
        per[short(r[h.index("Kernel Name")])].append(r)
    for k, rs in per.items():
        r = rs[0]
        lines.append(f"## `{k}`  ({len(rs)} launch(es) captured; first shown)")
        lines.append("")
        lines.append("| metric | value | unit |")
        lines.append("|---|---|---|")
        for m in KEY_METRICS:
            if m in h:
                i = h.index(m)
                lines.append(f"| {m} | {r[i]} | {units[i]} |")
        lines.append("")
        try:
            rd = float(r[h.index("dram__bytes_read.sum")].replace(",", ""))
            wr = float(r[h.index("dram__bytes_write.sum")].replace(",", ""))
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            rd *= scale.get(units[h.index("dram__bytes_read.sum")], 1)
            wr *= scale.get(units[h.index("dram__bytes_write.sum")], 1)
            base = k.split("<")[0]
            traffic[base] = rd + wr
        except (ValueError, KeyError):
            pass
    with open(os.path.join(PROF, f"{tag}_ncu_full.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    # per kernel: the utilisation of the resources that can bind it (bench.py quotes them beside
    # the roofline fraction)
    binding = {}
    pick = {"l1tex_data_pipe_pct": "l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed",
            "shared_wavefronts_pct": "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
            "l2_red_sectors_pct": "lts__t_sectors_srcunit_tex_op_red.sum.pct_of_peak_sustained_elapsed",
            "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "fp64_pipe_pct": "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
            "dram_pct": "dram__throughput.avg.pct_of_peak_sustained_elapsed",
            "sm_cycles_active_avg": "sm__cycles_active.avg", "sm_cycles_active_max": "sm__cycles_active.max"}
    for k, rs in per.items():
        r = rs[0]
        d = {}
        for name, m in pick.items():
            if m in h:
                try:
                    d[name] = float(r[h.index(m)].replace(",", ""))
                except ValueError:
                    pass
        binding[k.split("<")[0]] = d
    with open(os.path.join(PROF, "ncu_binding.json"), "w") as f:
        json.dump({"source": f"profiles/{tag}_ncu_full.md", "kernels": binding}, f, indent=1)
    with open(traffic_p, "w") as f:
        json.dump(traffic, f, indent=1)
    print("\n".join(lines[:60]))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", required=True)
    ap.add_argument("--launches", default=None)
    ap.add_argument("--full", default=None)
    a = ap.parse_args()
    os.makedirs(PROF, exist_ok=True)
    lp = a.launches or os.path.join(ROOT, "gpurun_out", f"{a.tag}_launches.csv")
    fp = a.full or os.path.join(ROOT, "gpurun_out", f"{a.tag}_full.ncu-rep")
    if os.path.exists(lp):
        launches(lp, a.tag)
    if os.path.exists(fp):
        full(fp, a.tag)


if __name__ == "__main__":
    main()
