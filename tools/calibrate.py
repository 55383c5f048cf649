"""Derive the fc2 head calibration constants in synth/calibration.json.

Without SimNet's trained weights (OUT of scope) the random-init
network must still produce realistic latencies: mean fetch latency ~1 cycle
(CPI ~ 1) and completion ~20 cycles so that ~25-35 context rows are live
("more than 68% of the instructions are paddings").  This
script runs the ORACLE (fp64) on a mixed-phase synthetic trace, measures the
raw head outputs and rescales gain/bias per output, a few fixed-point
iterations because the inputs depend on the latencies.  Only oracle/ and
synth/ are called.  Usage: python tools/calibrate.py [ARCH ...]
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import oracle  # noqa: E402
import synth  # noqa: E402

TARGET_MEAN = np.array([1.3, 30.0, 2.0])
TARGET_STD = np.array([0.7, 10.0, 2.0])
ITERS = 20
N_PER_PHASE = {"M2": 150, "C3": 120, "RB7": 60}


SEEDS = (synth.TRACE_SEED_BASE + 99, 31337)


def mixed_trace(n_per):
    """8 independent sub-traces: 4 phase epochs x 2 seeds (simulated with N = 8, W = 0)."""
    parts = [synth.trace(n_per, sd, r0=e * 262144 + 1000) for sd in SEEDS for e in range(4)]
    return np.concatenate(parts)


def main(archs):
    path = os.path.join(os.path.dirname(synth.__file__), "calibration.json")
    cal = json.load(open(path)) if os.path.exists(path) else {}
    for name in archs:
        arch, sparse = name.split(":")[0], name.endswith(":24")   # "<arch>:24" = the 2:4-pruned model
        tr = mixed_trace(N_PER_PHASE[arch])
        gain, bias = np.ones(3), np.zeros(3)
        for it in range(ITERS):
            w = synth.weights(arch, gain=gain, bias=bias, sparse24=sparse)
            r = oracle.simulate(tr, 8, 0, arch=arch, weights=w)
            y = r["y"].astype(np.float64)
            z = (y - bias) / gain                      # head output at gain 1, bias 0
            g_prev = gain.copy()
            if it == 0:                                # first: standardise the empty-context outputs
                gain = TARGET_STD / np.maximum(z.std(0), 1e-9) * 0.05
                bias = TARGET_MEAN - gain * z.mean(0)
            else:                                      # damped fixed point (feedback through the queue)
                gain = gain * np.clip(TARGET_STD / np.maximum(y.std(0), 1e-9), 0.5, 2.0) ** 0.5
                bias = bias + 0.5 * (TARGET_MEAN - y.mean(0))
            # completion (R21): bias fixed at COMPLETE_BIAS, non-negative row; the gain sets the mean
            o, b0 = synth.FLOOR_OUTPUT, synth.COMPLETE_BIAS
            if arch not in synth.FLOOR_ARCHS:
                o = None
            zf = None if o is None else (y[:, o] - b0) / g_prev[o]   # non-negative part at gain 1
            if o is not None:
                gain[o] = (TARGET_MEAN[o] - b0) / max(zf.mean(), 1e-9) if it == 0 else \
                    g_prev[o] * np.clip((TARGET_MEAN[o] - b0) / max(y[:, o].mean() - b0, 1e-9), 0.5, 2.0) ** 0.5
                bias[o] = b0
            lat = r["lat"].astype(np.float64)
            print(f"{name} it{it}: y mean {y.mean(0).round(3)} std {y.std(0).round(3)} | "
                  f"lat mean {lat.mean(0).round(3)} | k mean {r['k'].mean():.1f} max {r['k'].max()}"
                  f" | stalls {r['stalls']}", flush=True)
        cal[name] = {"gain": gain.tolist(), "bias": bias.tolist(),
                     "target_mean": TARGET_MEAN.tolist(), "target_std": TARGET_STD.tolist()}
        json.dump(cal, open(path, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1:] or ["M2", "C3", "RB7"])
