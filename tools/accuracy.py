"""Partitioning error vs the unpartitioned run (the Fig. 8 / Fig. 15 analog,
PAPER.md:201, :213, :221) on the GPU path: total cycles of an N-way partition
with warm-up W, with and without post-error correction (limit 100, :291),
relative to the same simulator at N = 1.  Synthetic SPEC-like trace, random-init
calibrated C3 weights (R12), bf16.

    python tools/accuracy.py [--L 200000] [--out profiles/r01_accuracy.json]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_pandeylfhl22_b200 as P  # noqa: E402
import synth  # noqa: E402


def run(tr, N, W, limit, w):
    with P.Simulator(precision="bf16", correction_limit=limit) as sim:
        sim.load_trace(tr)
        sim.partition(N, W)
        sim.load_model("C3", w)
        t0 = time.time()
        sim.simulate()
        st = sim.stats()
        return sim.total_cycles(), st["corrected"], time.time() - t0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--L", type=int, default=200_000)
    ap.add_argument("--seed", type=int, default=synth.TRACE_SEED_BASE + 1)
    ap.add_argument("--out", default="profiles/r01_accuracy.json")
    ap.add_argument("--config4", action="store_true",
                    help="BASELINE.json config 4: L = 10M (seed 20221113 + 4), N in 256..262144, "
                         "W in {0, 128, 1000, 10000}, no correction")
    a = ap.parse_args()
    if a.config4:
        return config4(a)
    tr = synth.trace(a.L, a.seed)
    w = synth.weights("C3")
    ref, _, t_ref = run(tr, 1, 0, 0, w)
    rows = []
    for N in (256, 1024, 4096):
        for W in (0, 10, 50, 110):
            for limit in (0, 100):
                tot, corr, t = run(tr, N, W, limit, w)
                rows.append(dict(N=N, W=W, correction=limit, total=tot, err=(tot - ref) / ref, corrected_rows=corr))
                print(f"N={N:5d} W={W:4d} corr={limit:3d}: err {100 * (tot - ref) / ref:+.3f}%  "
                      f"re-simulated rows {corr}", flush=True)
    res = dict(L=a.L, seed=a.seed, unpartitioned_total=ref, unpartitioned_seconds=t_ref, runs=rows,
               note="GPU bf16 C3 path; error = (total_N - total_1) / total_1 on the same simulator")
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(res, open(a.out, "w"), indent=1)


def config4(a):
    """Config 4 (the Fig. 6 analog): partition / warm-up sweep on a
    10M-instruction trace; error against the same GPU simulator at N = 1 (the unpartitioned
    CPU oracle would need ~1e14 FLOP single-threaded; the GPU path agrees with it to ~1e-5
    on the S3 parity cases)."""
    L = a.L if a.L != 200_000 else 10_000_000
    seed = synth.TRACE_SEED_BASE + 4
    tr = synth.trace(L, seed)
    w = synth.weights("C3")
    ref, _, t_ref = run(tr, 1, 0, 0, w)
    print(f"unpartitioned: total {ref} in {t_ref:.1f} s", flush=True)
    rows = []
    for N in [256 << i for i in range(11) if (256 << i) * 8 <= L]:
        for W in (0, 128, 1000, 10000):
            tot, _, t = run(tr, N, W, 0, w)
            rows.append(dict(N=N, W=W, total=tot, err=(tot - ref) / ref, seconds=t))
            print(f"N={N:6d} W={W:5d}: err {100 * (tot - ref) / ref:+.3f}%  ({t:.1f} s)", flush=True)
    res = dict(config=4, L=L, seed=seed, unpartitioned_total=ref, unpartitioned_seconds=t_ref, runs=rows,
               note="GPU bf16 C3 path; error = (total_N - total_1) / total_1 on the same simulator; no correction")
    out = a.out if a.out != "profiles/r01_accuracy.json" else "profiles/r01_config4_sweep.json"
    os.makedirs(os.path.dirname(out), exist_ok=True)
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
