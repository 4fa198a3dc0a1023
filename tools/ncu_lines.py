#!/usr/bin/env python
"""Per-CUDA-line hot spots of one kernel from an ncu report captured with --import-source on.

  python tools/ncu_lines.py REPORT.ncu-rep KERNEL_REGEX [--top N] [--sort inst|samples]

Prints, for the kernel's CUDA source lines (inlined device functions included), the warp
instructions executed, the stall samples and the shared-memory wavefronts, largest first.
"""
import csv
import io
import subprocess
import sys


def main():
    rep, kern = sys.argv[1], sys.argv[2]
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 40
    key = sys.argv[sys.argv.index("--sort") + 1] if "--sort" in sys.argv else "inst"
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--kernel-name", f"regex:{kern}", "--launch-count", "1"],
                         capture_output=True, text=True).stdout
    rows, path, hdr = [], "", None
    for rec in csv.reader(io.StringIO(out)):
        if not rec:
            continue
        if rec[0] == "File Path":
            path = rec[1].rsplit("/", 1)[-1]
        elif rec[0] == "Line No":
            hdr = rec
        elif hdr and rec[0] and rec[0].isdigit():
            d = dict(zip(hdr[2:], rec[2:]))  # duplicated 'Source' header: skip the first two columns
            def num(k):
                try:
                    return float(d.get(k, "0") or 0)
                except ValueError:
                    return 0.0
            rows.append((path, int(rec[0]), rec[1].strip()[:90], num("Instructions Executed"),
                         num("Warp Stall Sampling (All Samples)"), num("L1 Wavefronts Shared"),
                         num("Avg. Threads Executed")))
    tot_i = sum(r[3] for r in rows) or 1
    tot_s = sum(r[4] for r in rows) or 1
    idx = 3 if key == "inst" else 4
    print(f"total warp instructions {tot_i:.4g}, stall samples {tot_s:.4g}")
    print(f"{'file:line':28} {'inst%':>6} {'smpl%':>6} {'shwf':>10} {'thr':>5}  source")
    for r in sorted(rows, key=lambda r: -r[idx])[:top]:
        print(f"{r[0] + ':' + str(r[1]):28} {100 * r[3] / tot_i:6.2f} {100 * r[4] / tot_s:6.2f} {r[5]:10.4g} {r[6]:5.1f}  {r[2]}")


if __name__ == "__main__":
    main()
