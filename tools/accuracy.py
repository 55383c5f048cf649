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
                    help="BASELINE.json config 4: L = 10M (seed 20221113 + 3), N in 256..262144, "
                         "W in {0, 128, 1000, 10000}, no correction")
    ap.add_argument("--oracle-ref", default="profiles/r02_oracle_unpartitioned_c4_10M.json",
                    help="cached unpartitioned oracle run (tools/oracle_unpartitioned.py) for --config4")
    ap.add_argument("--s4", action="store_true", help="stage S4 at config 3 (100M rows, N = 65536, W = 110)")
    a = ap.parse_args()
    if a.config4:
        return config4(a)
    if a.s4:
        return s4(a)
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
    """Config 4 (the Fig. 6 analog): partition / warm-up sweep on the
    10M-instruction config-4 trace (seed 20221113 + 3: configs are numbered from 0 in the
    seed, as in bench.py).  Error of every partitioned GPU total against the UNPARTITIONED
    ORACLE (cached by tools/oracle_unpartitioned.py, bf16-operand mode) and against the
    same GPU simulator at N = 1."""
    L = a.L if a.L != 200_000 else 10_000_000
    seed = synth.TRACE_SEED_BASE + 3
    tr = synth.trace(L, seed)
    w = synth.weights("C3")
    oref = None
    if a.oracle_ref and os.path.exists(a.oracle_ref):
        o = json.load(open(a.oracle_ref))
        assert o["trace_seed"] == seed and o["rows"] >= L, (o["trace_seed"], o["rows"])
        oref = o["total"] if o["rows"] == L else o["clock_every"][L // o["every"] - 1]
    ref, _, t_ref = run(tr, 1, 0, 0, w)
    print(f"GPU unpartitioned: total {ref} in {t_ref:.1f} s; oracle unpartitioned {oref}"
          + (f" (GPU N=1 vs oracle {100 * (ref - oref) / oref:+.4f}%)" if oref else ""), flush=True)
    rows = []
    for N in [256 << i for i in range(11) if (256 << i) * 8 <= L]:
        for W in (0, 128, 1000, 10000):
            tot, _, t = run(tr, N, W, 0, w)
            r = dict(N=N, W=W, total=tot, err_vs_gpu_n1=(tot - ref) / ref, seconds=t)
            if oref:
                r["err_vs_oracle"] = (tot - oref) / oref
            rows.append(r)
            print(f"N={N:6d} W={W:5d}: err vs GPU N=1 {100 * (tot - ref) / ref:+.3f}%"
                  + (f", vs oracle {100 * (tot - oref) / oref:+.3f}%" if oref else "") + f"  ({t:.1f} s)", flush=True)
    # S4 at config 3's partition geometry (sub-traces of 1526 rows, W = 110 = Context_length) on this
    # trace, where the unpartitioned ORACLE reference exists: N = L / 1526, with and without post-error
    # correction (limit 100)
    s4 = []
    N3 = L // (100_000_000 // 65536)
    for limit in (0, 100):
        tot, corr, t = run(tr, N3, 110, limit, w)
        r = dict(N=N3, W=110, correction_limit=limit, total=tot, corrected_rows=corr,
                 err_vs_gpu_n1=(tot - ref) / ref, seconds=t)
        if oref:
            r["err_vs_oracle"] = (tot - oref) / oref
        s4.append(r)
        print(f"S4 geometry N={N3} W=110 limit={limit}: err vs GPU N=1 {100 * (tot - ref) / ref:+.4f}%"
              + (f", vs oracle {100 * (tot - oref) / oref:+.4f}%" if oref else ""), flush=True)
    res = dict(config=4, L=L, seed=seed, gpu_unpartitioned_total=ref, gpu_unpartitioned_seconds=t_ref,
               oracle_unpartitioned_total=oref, oracle_ref=a.oracle_ref, runs=rows, s4_geometry=s4,
               note="GPU bf16 C3 path, no correction; errors signed, (total_N - reference) / reference")
    out = a.out if a.out != "profiles/r01_accuracy.json" else "profiles/r02_config4_sweep.json"
    os.makedirs(os.path.dirname(out), exist_ok=True)
    json.dump(res, open(out, "w"), indent=1)


def s4(a):
    """Stage S4 at the bench workload (config 3: 100M instructions, N = 65536, W = 110, C3,
    bf16): partitioned total vs the unpartitioned (N = 1) run of the same GPU simulator over
    all 100M rows (the unpartitioned CPU oracle at 1e8 sequential C3 steps is out of reach:
    ~45 h single-threaded; the link GPU N = 1 == oracle N = 1 is established on the 10M-row
    config-4 trace by config4()).  Also with post-error correction (limit 100)."""
    L, N, W = 100_000_000, 65536, 110
    seed = synth.TRACE_SEED_BASE + 2
    tr = synth.trace(L, seed)
    w = synth.weights("C3")
    ref, _, t_ref = run(tr, 1, 0, 0, w)
    print(f"GPU unpartitioned: total {ref} in {t_ref:.1f} s", flush=True)
    rows = []
    for limit in (0, 100):
        tot, corr, t = run(tr, N, W, limit, w)
        rows.append(dict(N=N, W=W, correction_limit=limit, total=tot, corrected_rows=corr,
                         err=(tot - ref) / ref, seconds=t))
        print(f"N={N} W={W} limit={limit}: total {tot} err {100 * (tot - ref) / ref:+.4f}% ({t:.1f} s)", flush=True)
    res = dict(stage="S4", config=3, L=L, seed=seed, unpartitioned_total=ref, unpartitioned_seconds=t_ref,
               runs=rows, criterion="|err| <= 0.5% (north_star)")
    out = a.out if a.out != "profiles/r01_accuracy.json" else "profiles/r02_s4_config3.json"
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
