"""Host-side pieces of bench.py (CPU): the multi-threaded oracle timing leg computes the same
histograms as the single-threaded oracle (it only shards the work and sums per-thread histograms
in fixed order, S§8(d)), and the reference arm's JSON line keeps the driver contract."""
import json
import os
import subprocess
import sys

import numpy as np

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def test_threaded_oracle_equals_single_thread():
    import bench
    wl = synth.make_workload("tiny")
    ev = synth.events_for_run(wl, 0)
    onorm, obm, _ = oracle.run_workload(wl, events={0: ev})
    for threads, stride in ((1, 1), (3, 1), (4, 1)):
        _, _, norm, bm = bench.oracle_timed(wl, ev, stride, threads)
        assert np.allclose(norm, onorm, rtol=1e-13, atol=0)
        assert np.array_equal(bm, obm)  # unit weights: exact counts in any order


def test_reference_arm_line(tmp_path):
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                        "--warmup", "0", "--ref-stride", "16"], capture_output=True, text=True, env=env,
                       timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["e2e"]["unit"] == line["unit"]
