"""Run the RB7 CNN (stem, fused residual blocks, fc1, head) on the same inputs several times
through psim_cnn_forward and report which sub-traces' outputs differ between runs
(diagnosis of the residual-block ordering bug; PSIM_LIB selects the build)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import paper_conf_sc_pandeylfhl22_b200 as P  # noqa: E402
import synth  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 40000
rng = np.random.default_rng(5)
X = np.zeros((B, 112, 50), np.float32)
k = rng.integers(0, 110, B)
for b in range(B):
    X[b, : k[b] + 1, 3:] = rng.integers(0, 256, (k[b] + 1, 47))
    X[b, 1 : k[b] + 1, :3] = rng.integers(0, 200, (k[b], 3))
w = synth.weights("RB7")
outs = []
with P.Simulator(precision="bf16") as sim:
    sim.load_model("RB7", w)
    for r in range(4):
        outs.append(sim.cnn_forward(X))
base = outs[0]
for r in range(1, 4):
    d = np.nonzero(np.any(outs[r] != base, axis=1))[0]
    print(f"run {r}: {len(d)} of {B} sub-traces differ;", "b % 2:", np.bincount(d % 2, minlength=2).tolist(),
          "first:", d[:12].tolist(), "max |dy|:", float(np.max(np.abs(outs[r] - base))) if len(d) else 0.0)
