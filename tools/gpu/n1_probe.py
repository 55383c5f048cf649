# N = 1 vs N = 4 with full warm-up (W >= s_j => partitioned == unpartitioned, bit-exact) on the CNN path
import sys, numpy as np, paper_conf_sc_pandeylfhl22_b200 as P, synth
w = synth.weights("C3")
for L in (100_000, 300_000, 1_000_000):
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 4)
    out = []
    for N, W in ((1, 0), (4, L), (64, 0), (64, 2000)):
        with P.Simulator(precision="bf16") as sim:
            sim.load_trace(tr); sim.partition(N, W); sim.load_model("C3", w); sim.simulate()
            out.append((N, W, sim.total_cycles(), sim.stats()["k_hist"][:3]))
    print(L, [(n, wv, t) for n, wv, t, _ in out], flush=True)
