"""The synthetic model has no frozen-Clock fixed point (R21).

Round 1's random-weight model fell, at row ~3.3M of the config-4 trace, into a state
where it predicted f = c = s = 0 with an unchanging context for millions of rows (the
Clock never advanced, so nothing retired and the next input was the same).  R21 removes
it by construction: the completion row of the fc2 head is non-negative with a bias
> 0.5, so every predicted completion latency is >= 1.  Pins:

* the construction itself on the weight files both sides load (every arch);
* the consequence for the queue rules, independent of any CNN: with c >= 1 the Clock
  cannot stay still for more than Context_length consecutive instructions, because each
  one pushes an entry that is still live and the ROB-full stall (R5)
  advances the Clock once the queue holds more than 110 -- checked on adversarial
  teacher-forced latencies (f = 0 always) where the bound is reached exactly;
* the oracle's CNN runs: c >= 1 on every row, and the longest zero-advance run is short.
"""
import numpy as np
import pytest

import oracle
import synth


@pytest.mark.parametrize("arch", list(synth.FLOOR_ARCHS))
def test_completion_row_nonnegative_with_bias_above_half(arch):
    w = synth.weights(arch)
    shapes = synth.layer_shapes(arch)
    n_head = int(np.prod(shapes[-1][0])) + int(np.prod(shapes[-1][1]))
    head_w = w[-n_head:-3].reshape(shapes[-1][0])
    head_b = w[-3:]
    assert np.all(head_w[synth.FLOOR_OUTPUT] >= 0)
    assert head_b[synth.FLOOR_OUTPUT] > 0.5
    # the other outputs keep signed weights (context-dependent fetch / store latencies)
    assert np.any(head_w[0] < 0) and np.any(head_w[2] < 0)


def _longest_zero_advance_run(clock):
    adv = np.diff(np.concatenate([[0], clock])) == 0
    best = cur = 0
    for a in adv:
        cur = cur + 1 if a else 0
        best = max(best, cur)
    return best


@pytest.mark.parametrize("cap", [4, 17, 110])
def test_zero_advance_runs_bounded_by_capacity(cap):
    """f = 0 for every instruction, c >= 1: the Clock advances only through ROB-full
    stalls; no run of instructions without a Clock advance is longer than the capacity."""
    L = 3000
    tr = synth.trace(L, 5)
    lat = synth.teacher_latencies(L, 11, c_mean=50.0)
    lat[:, 0] = 0
    lat[:, 1] = np.maximum(lat[:, 1], 1)
    r = oracle.simulate(tr, 1, 0, forced_lat=lat, cap=cap)
    run = _longest_zero_advance_run(r["clock"])
    assert run <= cap
    assert run == cap          # the bound is attained (the stall fires exactly at cap + 1 entries)
    assert r["stalls"] > 0


@pytest.mark.parametrize("arch,mode", [("C3", oracle.FP64), ("C3", oracle.BF16)])
def test_model_completion_floor_and_clock_progress(arch, mode):
    L = 2500
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 3)
    w = synth.weights(arch)
    r = oracle.simulate(tr, 1, 0, arch=arch, weights=w, mode=mode)
    assert r["lat"][:, 1].min() >= 1
    assert np.all(r["y"][:, 1] >= 0.5)
    assert _longest_zero_advance_run(r["clock"]) <= 110
    cpi = r["total"] / L
    assert 0.5 < cpi < 3.0
    assert 5 < r["k"].mean() < 60
