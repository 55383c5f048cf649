"""Pins of the oracle's post-error correction (PAPER.md:203-219 [V-B], Fig. 9,
limit :291; R19), independent of its implementation:

* N = 2, W = 0: sub-trace 0 starts from the empty queue at row 0 exactly like
  the unpartitioned run, so its re-simulation of sub-trace 1's rows IS the
  unpartitioned (N = 1) trajectory.  The stop row is then the first row of
  sub-trace 1 where the N = 1 and N = 2 runs see the same context count, and
  the corrected cycles are the per-row clock advances of the N = 1 run before
  the stop row plus those of the N = 2 run after it -- all read from two plain
  oracle.simulate runs.
* W >= s_j: every first pass already starts from row 0, so the counts match at
  once and nothing is corrected.
* Fig. 9 rank rule: the first sub-trace of every GPU is never corrected.
* limit 0 = no correction; first-pass cycles = oracle.simulate's.
"""
import numpy as np
import pytest

import oracle
import synth


def _expected_n2(tr, lat, limit, cap, arch="C3", weights=None, mode=oracle.FP64):
    L = tr.shape[0]
    kw = dict(forced_lat=lat, cap=cap, arch=arch, weights=weights, mode=mode)
    u = oracle.simulate(tr, 1, 0, **kw)
    f = oracle.simulate(tr, 2, 0, **kw)
    s1 = L // 2
    r = s1
    while r < L and r - s1 < limit and u["k"][r] != f["k"][r]:
        r += 1
    adv_u = np.diff(np.concatenate([[0], u["clock"]]))          # per-row Clock advance, N = 1
    adv_f = np.diff(np.concatenate([[0], f["clock"][s1:]]))       # sub-trace 1 starts at Clock 0
    cyc1 = int(adv_u[s1:r].sum() + adv_f[r - s1:].sum())
    return r, cyc1, u, f


@pytest.mark.parametrize("limit", [100, 7, 1, 10**6])
@pytest.mark.parametrize("cap", [4, 110])
def test_n2_correction_equals_unpartitioned_prefix_forced(limit, cap):
    L = 3001
    tr = synth.trace(L, 11)
    lat = synth.teacher_latencies(L, 3, big=0.05)
    r, cyc1, u, f = _expected_n2(tr, lat, limit, cap)
    o = oracle.simulate_pec(tr, 2, 0, limit=limit, forced_lat=lat, cap=cap)
    s1 = L // 2
    assert o["corr_len"][0] == 0 and o["corr_len"][1] == r - s1
    assert o["cycles"][0] == f["cycles"][0]
    assert o["cycles"][1] == cyc1
    assert np.array_equal(o["cycles1"], f["cycles"])
    assert np.array_equal(o["corr_lat"][s1:r], u["lat"][s1:r])
    assert np.array_equal(o["corr_k"][s1:r], u["k"][s1:r])
    assert np.all(o["corr_k"][r:] == -1) and np.all(o["corr_k"][:s1] == -1)


def test_n2_correction_stalls_exercised():
    # cap 4 with 5 % long latencies: the corrected rows include ROB-full stalls,
    # so a wrong Clock bookkeeping in the replacement cannot cancel out
    L = 3001
    tr = synth.trace(L, 11)
    lat = synth.teacher_latencies(L, 3, big=0.05)
    r, cyc1, u, f = _expected_n2(tr, lat, 10**6, 4)
    assert r > L // 2
    assert cyc1 != f["cycles"][1]                 # the correction changes the answer


@pytest.mark.parametrize("mode", [oracle.FP64, oracle.BF16])
def test_n2_correction_equals_unpartitioned_prefix_cnn(mode):
    L = 1201
    tr = synth.trace(L, 4)
    w = synth.weights("C3")
    r, cyc1, u, f = _expected_n2(tr, None, 100, 110, weights=w, mode=mode)
    o = oracle.simulate_pec(tr, 2, 0, limit=100, weights=w, mode=mode)
    assert o["corr_len"][1] == r - L // 2 > 0
    assert o["cycles"][1] == cyc1
    assert np.array_equal(o["corr_lat"][L // 2:r], u["lat"][L // 2:r])


def test_full_warmup_needs_no_correction():
    L, N = 900, 6
    tr = synth.trace(L, 2)
    lat = synth.teacher_latencies(L, 1, big=0.05)
    o = oracle.simulate_pec(tr, N, L, limit=100, forced_lat=lat, cap=8)
    assert np.all(o["corr_len"] == 0)
    assert o["total"] == o["total1"] == oracle.simulate(tr, 1, 0, forced_lat=lat, cap=8)["total"]


def test_fig9_first_partition_of_each_gpu_not_corrected():
    # "20 instructions are partitioned into four sub-traces and simulated on two
    # GPUs ... partitions 0 and 2 re-simulate ... from partitions 1 and 3"
    L, N = 20, 4
    tr = synth.trace(L, 9)
    lat = synth.teacher_latencies(L, 9, big=0.3)
    one = oracle.simulate_pec(tr, N, 0, limit=100, G=1, forced_lat=lat, cap=3)
    two = oracle.simulate_pec(tr, N, 0, limit=100, G=2, forced_lat=lat, cap=3)
    four = oracle.simulate_pec(tr, N, 0, limit=100, G=4, forced_lat=lat, cap=3)
    assert two["corr_len"][0] == 0 and two["corr_len"][2] == 0       # first on GPU 0 / GPU 1
    assert two["corr_len"][1] == one["corr_len"][1] and two["corr_len"][3] == one["corr_len"][3]
    assert two["cycles"][3] == one["cycles"][3] and two["cycles"][2] == one["cycles1"][2]
    assert np.all(four["corr_len"] == 0) and four["total"] == four["total1"]
    assert one["corr_len"][1] + one["corr_len"][2] + one["corr_len"][3] > 0


def test_limit_zero_is_first_pass_and_limit_bounds():
    L, N = 4000, 16
    tr = synth.trace(L, 5)
    lat = synth.teacher_latencies(L, 5, big=0.05)
    base = oracle.simulate(tr, N, 3, forced_lat=lat, cap=6)
    o0 = oracle.simulate_pec(tr, N, 3, limit=0, forced_lat=lat, cap=6)
    assert np.array_equal(o0["cycles"], base["cycles"]) and np.all(o0["corr_len"] == 0)
    o5 = oracle.simulate_pec(tr, N, 3, limit=5, forced_lat=lat, cap=6)
    assert np.array_equal(o5["cycles1"], base["cycles"])
    assert o5["corr_len"].max() <= 5 and o5["corr_len"][0] == 0
    # a sampled range [j0, j0+nj) corrects only inside the range
    full = oracle.simulate_pec(tr, N, 3, limit=50, forced_lat=lat, cap=6)
    part = oracle.simulate_pec(tr, N, 3, limit=50, forced_lat=lat, cap=6, j0=5, nj=4)
    assert part["corr_len"][0] == 0
    assert np.array_equal(part["cycles"][1:], full["cycles"][6:9])


def test_correction_reduces_cnn_partition_error():
    # PAPER.md:219/Fig. 15: post-error correction reduces the error of small-warm-up runs
    L, N = 2400, 24
    tr = synth.trace(L, 7)
    w = synth.weights("C3")
    ref = oracle.simulate(tr, 1, 0, weights=w, want_rows=False)["total"]
    o = oracle.simulate_pec(tr, N, 0, limit=100, weights=w, want_rows=False)
    assert abs(o["total"] - ref) < abs(o["total1"] - ref)
