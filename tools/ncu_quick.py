#!/usr/bin/env python
"""Run a command under ncu with a few metrics and print one line per kernel launch.

  python tools/ncu_quick.py [--metrics m1,m2] [--filter regex] -- cmd ...
(on the GPU box; never under a multi-rank command)
"""
import csv
import io
import re
import subprocess
import sys

DEFAULT = "gpu__time_duration.sum,sm__cycles_active.avg,sm__cycles_active.max"


def main():
    argv = sys.argv[1:]
    metrics, filt = DEFAULT, ""
    while argv and argv[0] != "--":
        if argv[0] == "--metrics":
            metrics = argv[1]
            argv = argv[2:]
        elif argv[0] == "--filter":
            filt = argv[1]
            argv = argv[2:]
        else:
            raise SystemExit(f"unknown option {argv[0]}")
    cmd = ["ncu", "--metrics", metrics, "--clock-control", "none", "--csv"] + argv[1:]
    out = subprocess.run(cmd, capture_output=True, text=True).stdout
    lines = [ln for ln in out.splitlines() if ln.startswith('"')]
    rows = list(csv.reader(io.StringIO("\n".join(lines))))
    if not rows:
        print(out[-2000:])
        return
    hdr = rows[0]
    launches = {}
    for r in rows[1:]:
        d = dict(zip(hdr, r))
        name = re.sub(r"\(.*", "", d["Kernel Name"])[:60]
        if filt and not re.search(filt, d["Kernel Name"]):
            continue
        key = (d["ID"], name, d.get("Grid Size", ""))
        launches.setdefault(key, {})[d["Metric Name"]] = d["Metric Value"]
    for (i, name, grid), ms in launches.items():
        print(i, name, grid, " ".join(f"{k}={v}" for k, v in ms.items()))


if __name__ == "__main__":
    main()
