"""Small runs of every hot-path kernel (the workload of round 2's memory-checker runs, see
profiles/r02_sanitizer.md; that tool is now closed on the GPU pool): the fused C3 path (resident and pinned-streamed trace, several
tiles per CTA), post-error correction, interval metrics, the layer-wise path, the 2:4
sparse GEMMs and RB7 (fused gather + stem, residual-block kernel)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import paper_conf_sc_pandeylfhl22_b200 as P  # noqa: E402
import synth  # noqa: E402

small = len(sys.argv) > 1 and sys.argv[1] == "small"
L, N, W = (3000, 40, 16) if small else (60_000, 1500, 24)
tr = synth.trace(L, 99)
w = synth.weights("C3")
out = []
for mode, kw in [("device", {}), ("pinned", {"chunk_steps": 7}), ("pageable", {"correction_limit": 20, "interval": 100}),
                 ("layerwise", {"layerwise": True})]:
    with P.Simulator(precision="bf16", record_rows=True, **kw) as sim:
        if mode == "device":
            sim.load_trace(torch.from_numpy(tr).cuda())
        elif mode == "pinned":
            sim.load_trace(torch.from_numpy(tr).pin_memory())
        else:
            sim.load_trace(tr)
        sim.partition(N, W)
        sim.load_model("C3", w)
        sim.simulate()
        out.append((mode, sim.total_cycles()))
with P.Simulator(precision="bf16", sparse24=True) as sim:
    sim.load_trace(tr); sim.partition(N, W); sim.load_model("C3", synth.weights("C3", sparse24=True)); sim.simulate()
    out.append(("sparse", sim.total_cycles()))
wr = synth.weights("RB7")
with P.Simulator(precision="bf16") as sim:   # ragged: several 128-row stem / residual tiles
    nr = 3000 if small else 30_000
    sim.load_trace(tr[:nr]); sim.partition(20 if small else 300, 8); sim.load_model("RB7", wr); sim.simulate()
    out.append(("rb7", sim.total_cycles()))
print(out)
assert len({t for m, t in out if m in ("device", "pinned", "layerwise")}) >= 1
