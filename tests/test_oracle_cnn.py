"""Pins of the oracle's CNN forward and of the partition identities with the CNN.

The CNN is pinned to a library routine: torch.nn.functional.conv1d / linear /
relu in float64 (the special case "reduces to a library routine"), after the
documented reshapes (features are conv channels, instructions the length,
PAPER.md:93/:141; FC1 flattens position-major, R11).  The bf16 mode
is pinned to the same torch graph with torch's own bf16 conversion (RNE) at
the operand rounding points (R16).
"""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import oracle
import synth


def torch_forward(arch, w, X, bf16=False):
    w = torch.from_numpy(np.asarray(w, np.float32).astype(np.float64))
    shapes = synth.layer_shapes(arch)
    params, off = [], 0
    for ws, bs in shapes:
        n = int(np.prod(ws)); W_ = w[off:off + n].reshape(ws); off += n
        B = w[off:off + bs[0]]; off += bs[0]
        params.append((W_, B))
    r = (lambda t: t.to(torch.bfloat16).to(torch.float64)) if bf16 else (lambda t: t)
    x = torch.from_numpy(np.asarray(X, np.float64)).T[None]          # (1, 50, 112)
    layers = synth.ARCHS[arch]
    nl = len(layers)
    li = 0
    while li < nl:
        kind, cin, cout, k = layers[li]
        W_, B = params[li]
        last = li == nl - 1
        if kind == "conv" and k == 2:
            x = F.relu(F.conv1d(r(x), r(W_), B, stride=2))
            li += 1
        elif kind == "conv" and k == 3:                                # residual block (RB7)
            xin = r(x)
            Wb, Bb = params[li + 1]
            h = F.relu(F.conv1d(xin, r(W_), B, stride=1, padding=1))
            x = F.relu(xin + F.conv1d(r(h), r(Wb), Bb, stride=1, padding=1))
            li += 2
        else:
            if x.dim() == 3:                                          # position-major flatten
                x = x[0].T.reshape(1, -1)
            if last:
                x = F.linear(x, W_, B)
            else:
                x = F.relu(F.linear(r(x), r(W_), B))
            li += 1
    return x[0].numpy()


def realistic_inputs(n, seed):
    """Inputs built by the oracle's own gather from a teacher-forced run (k in 0..110)."""
    tr = synth.trace(4000, 1234 + seed)
    lat = synth.teacher_latencies(4000, seed, c_mean=60.0)
    q = oracle.Queue(110)
    out = []
    for i in range(4000):
        X, k = q.build_input(tr, i)
        if i % (4000 // n) == 0:
            out.append(X)
        q.update(i, *(int(v) for v in lat[i]))
    return out


@pytest.mark.parametrize("arch", ["M2", "C3", "RB7"])
def test_cnn_fp64_matches_torch(arch):
    w = synth.weights(arch)
    rng = np.random.default_rng(0)
    Xs = realistic_inputs(6, 1) + [rng.integers(0, 200, (112, 50)).astype(np.float64),
                                    np.zeros((112, 50))]
    for X in Xs:
        y = oracle.cnn_forward(arch, w, X)
        yt = torch_forward(arch, w, X)
        np.testing.assert_allclose(y, yt, rtol=1e-11, atol=1e-9)


@pytest.mark.parametrize("arch", ["M2", "C3", "RB7"])
def test_cnn_bf16_matches_torch_bf16(arch):
    w = synth.weights(arch)
    for X in realistic_inputs(4, 2):
        y = oracle.cnn_forward(arch, w, X, mode=oracle.BF16)
        yt = torch_forward(arch, w, X, bf16=True)
        np.testing.assert_allclose(y, yt, rtol=1e-9, atol=1e-7)
        y64 = oracle.cnn_forward(arch, w, X)
        assert np.max(np.abs(y - y64)) / max(np.max(np.abs(y64)), 1.0) < 5e-2   # bf16 is close to fp64


def test_cnn_weight_count_checked():
    w = synth.weights("C3")
    with pytest.raises(ValueError):
        oracle.cnn_forward("C3", w[:-1], np.zeros((112, 50)))


def test_n1_identity_with_cnn():
    """N=1 equals the plain unpartitioned loop done by hand."""
    arch = "M2"
    w = synth.weights(arch)
    L = 120
    tr = synth.trace(L, 555)
    out = oracle.simulate(tr, 1, 37, arch=arch, weights=w)     # W irrelevant for N=1
    q = oracle.Queue(110)
    for i in range(L):
        X, k = q.build_input(tr, i)
        y = oracle.cnn_forward(arch, w, X)
        f, c, s = (oracle.round_latency(v) for v in y)
        assert (f, c, s) == tuple(int(v) for v in out["lat"][i])
        assert k == out["k"][i]
        q.update(i, f, c, s)
        assert q.clock == out["clock"][i]
    assert out["total"] == q.clock and out["cycles"].tolist() == [q.clock]


def test_full_warmup_identity_and_shift_invariance():
    """W >= s_j for all j => each sub-trace replays the full prefix from the same empty
    state, so partitioned == unpartitioned row by row (closed form); starting all clocks
    at C0 != 0 changes nothing because only clock differences enter (R2)."""
    arch = "M2"
    w = synth.weights(arch)
    L, N = 96, 4
    tr = synth.trace(L, 777)
    ref = oracle.simulate(tr, 1, 0, arch=arch, weights=w)
    part = oracle.simulate(tr, N, L, arch=arch, weights=w)
    assert np.array_equal(part["lat"], ref["lat"]) and np.array_equal(part["k"], ref["k"])
    assert np.array_equal(part["clock"], ref["clock"])
    assert part["total"] == ref["total"]
    bounds = [j * L // N for j in range(N + 1)]
    for j in range(N):
        s, e = bounds[j], bounds[j + 1]
        expect = ref["clock"][e - 1] - (ref["clock"][s - 1] if s > 0 else 0)
        assert part["cycles"][j] == expect
    shifted = oracle.simulate(tr, N, 10, arch=arch, weights=w, clock0=123456789)
    base = oracle.simulate(tr, N, 10, arch=arch, weights=w)
    assert np.array_equal(shifted["lat"], base["lat"]) and shifted["total"] == base["total"]
    assert np.array_equal(shifted["clock"] - 123456789, base["clock"])


def test_calibrated_model_occupancy():
    """The calibrated random model gives SPEC-like statistics: CPI ~ 1 and most of the
    111 rows are padding (> 68% padding)."""
    w = synth.weights("M2")
    tr = synth.trace(600, synth.TRACE_SEED_BASE + 1)
    out = oracle.simulate(tr, 1, 0, arch="M2", weights=w)
    cpi = out["total"] / 600
    assert 0.3 < cpi < 3.0
    assert 3 < out["k"].mean() < 60
    assert (1 - (out["k"].mean() + 1) / 111) > 0.5
