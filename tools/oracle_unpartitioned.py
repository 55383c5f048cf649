"""Unpartitioned (N = 1) oracle run over a prefix of a config's trace, cached as the
reference of the partition / warm-up sweep (config 4, Fig. 6) and of
the GPU's N = 1 runs.  Calls only oracle/ and synth/ (test infrastructure; no product
code).  Writes JSON: total cycles, stalls, and the Clock after every `--every`-th row
(so a prefix of the run is a reference for a shorter trace as well).

    python tools/oracle_unpartitioned.py --config 4 --rows 10000000 --mode bf16 \
        --out profiles/r02_oracle_unpartitioned_c4_10M.json
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import oracle  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4, help="BASELINE.json config id (trace seed = base + id - 1)")
    ap.add_argument("--rows", type=int, default=10_000_000)
    ap.add_argument("--arch", default="C3")
    ap.add_argument("--mode", default="bf16", choices=["bf16", "fp64"])
    ap.add_argument("--every", type=int, default=10_000)
    ap.add_argument("--out", required=True)
    a = ap.parse_args()
    seed = synth.TRACE_SEED_BASE + a.config - 1
    tr = synth.trace(a.rows, seed)
    w = synth.weights(a.arch)
    t0 = time.time()
    r = oracle.simulate(tr, 1, 0, arch=a.arch, weights=w, mode=oracle.BF16 if a.mode == "bf16" else oracle.FP64)
    dt = time.time() - t0
    clk = r["clock"]
    lat = r["lat"].astype(np.int64)
    zero = np.diff(np.concatenate([[0], clk])) == 0
    best = cur = 0
    for z in zero:
        cur = cur + 1 if z else 0
        best = max(best, cur)
    out = {"config": a.config, "trace_seed": seed, "rows": a.rows, "arch": a.arch, "mode": a.mode,
           "total": int(r["total"]), "stalls": int(r["stalls"]), "seconds": dt,
           "cpi": float(r["total"]) / a.rows, "k_mean": float(r["k"].mean()),
           "lat_mean": lat.mean(0).tolist(), "longest_zero_advance_run": int(best),
           "every": a.every, "clock_every": [int(x) for x in clk[a.every - 1::a.every]]}
    with open(a.out, "w") as f:
        json.dump(out, f)
    print(json.dumps({k: v for k, v in out.items() if k != "clock_every"}))


if __name__ == "__main__":
    main()
