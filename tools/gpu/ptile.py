import numpy as np, paper_conf_sc_pandeylfhl22_b200 as P, synth, torch
L, N, W = 10_000_000, 6554, 110   # config-3 per-sub-trace length (1526) on a 1/10 slice
tr = synth.trace(L, synth.TRACE_SEED_BASE + 3)
w = synth.weights("C3")
with P.Simulator(precision="bf16") as sim:
    sim.load_trace(torch.from_numpy(tr).cuda()); sim.partition(N, W); sim.load_model("C3", w); sim.simulate()
    st = sim.stats()
kh = np.array(st["k_hist"], dtype=np.float64)
k = np.arange(len(kh)); Pb = np.minimum((k + 8) // 8, 14)
print("mean k", (kh * k).sum() / kh.sum(), "mean P_b", (kh * Pb).sum() / kh.sum(), "mean P_tile", st["layer_k"][3] / 1000 / 128)
print("P_b histogram", [float(kh[Pb == p].sum() / kh.sum()) for p in range(1, 9)])
