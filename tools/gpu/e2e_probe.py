# where does the end-to-end (pinned host trace) run lose time against the device-resident run?
import time, numpy as np, torch, paper_conf_sc_pandeylfhl22_b200 as P, synth
L, N, W = 100_000_000, 65536, 110
host = torch.empty((L, 48), dtype=torch.uint8, pin_memory=True)
synth.trace_into(host.numpy(), synth.TRACE_SEED_BASE + 3, 0)
dev = host.cuda()
w = synth.weights("C3")
st = torch.cuda.Stream()
sim = P.Simulator(precision="bf16", stream=st.cuda_stream, profile=True)
sim.load_model("C3", w)
for name, tr in (("resident", dev), ("pinned", host)):
    sim.load_trace(tr, n_instr=L); sim.partition(N, W)
    sim.simulate(); torch.cuda.synchronize()
    t0 = time.time(); sim.simulate(); torch.cuda.synchronize(); wall = (time.time() - t0) * 1e3
    s = sim.stats()
    print(name, "wall %.1f ms" % wall, "sim_ms %.1f load_ms %.1f" % (s["sim_ms"], s["load_ms"]),
          "kernel_ms", [round(x, 1) for x in s["kernel_ms"]], "launches", list(s["kernel_launches"]))
