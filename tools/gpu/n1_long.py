# long single-sub-trace run: CPI per 250k-row window and per-window mean k (where does it drift?)
import numpy as np, paper_conf_sc_pandeylfhl22_b200 as P, synth
L = 10_000_000
tr = synth.trace(L, synth.TRACE_SEED_BASE + 4)
w = synth.weights("C3")
with P.Simulator(precision="bf16", record_rows=True) as sim:
    sim.load_trace(tr); sim.partition(1, 0); sim.load_model("C3", w); sim.simulate()
    lat, k, clk = sim.get_rows(0, L)
    print("total", sim.total_cycles(), "stalls", sim.stats()["stalls"])
clk = clk.astype(np.int64)
for s in range(0, L, 250_000):
    e = min(L, s + 250_000)
    c0 = clk[s - 1] if s else 0
    print(s, "CPI %.3f" % ((clk[e - 1] - c0) / (e - s)), "mean k %.1f" % k[s:e].mean(),
          "mean f %.2f c %.2f s %.2f" % tuple(lat[s:e].mean(axis=0)), flush=True)
