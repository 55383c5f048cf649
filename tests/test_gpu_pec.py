"""GPU parity of post-error correction (PAPER.md:203-219 [V-B], Fig. 9; DESIGN.md
R19) through the C ABI vs oracle.simulate_pec (pinned in test_oracle_pec.py).

S1  teacher-forced latencies: first-pass and corrected per-sub-trace cycles,
    re-simulated row counts, the re-simulation's (f, c, s) and context counts,
    totals -- bit-exact, on the warp-per-sub-trace update kernel and on the
    fused C3 kernels (PSIM_FORCE_PREDICT runs the CNN but follows the forced
    trajectory, so stop decisions are integer work).
S3  free-running bf16 C3 with correction: total within 0.5% of the bf16 oracle.
"""
import numpy as np
import pytest

import oracle
import paper_conf_sc_pandeylfhl22_b200 as P
import synth

pytestmark = pytest.mark.gpu


def pec_run(trace, N, W, limit, *, cap=110, forced=None, weights=None, force_predict=False, layerwise=False,
            rank=0, world=1, first_row=0, n_instr=None, record=True):
    with P.Simulator(precision="bf16", queue_cap=cap, record_rows=record, correction_limit=limit,
                     force_predict=force_predict, layerwise=layerwise, rank=rank, world_size=world) as sim:
        sim.load_trace(trace, n_instr=n_instr, first_row=first_row)
        sim.partition(N, W)
        if weights is not None:
            sim.load_model("C3", weights)
        if forced is not None:
            sim.force_latencies(forced)
        sim.simulate()
        rr = sim.rank_range()
        cl, c1 = sim.corrections()
        out = dict(total=sim.total_cycles(), cycles=sim.subtrace_cycles(), corr_len=cl, cycles1=c1,
                   stats=sim.stats(), rr=rr)
        if record and rr.j1 > rr.j0:
            L = n_instr if n_instr is not None else trace.shape[0]
            s0 = rr.j0 * L // N
            out["corr_lat"], out["corr_k"] = sim.get_corrected_rows(s0, rr.row_hi - s0)
            out["first"] = s0
        return out


def _check_s1(g, ref, lo=None, hi=None):
    lo = g["first"] if lo is None else lo
    hi = lo + len(g["corr_k"]) if hi is None else hi
    assert np.array_equal(g["cycles1"], ref["cycles1"])
    assert np.array_equal(g["corr_len"], ref["corr_len"])
    assert np.array_equal(g["cycles"], ref["cycles"])
    assert np.array_equal(g["corr_k"], ref["corr_k"][lo:hi])
    m = ref["corr_k"][lo:hi] >= 0
    assert np.array_equal(g["corr_lat"][m], ref["corr_lat"][lo:hi][m])
    assert g["stats"]["corrected"] == int(ref["corr_len"].sum())


@pytest.mark.parametrize("L,N,W,cap,limit,big", [
    (20, 4, 0, 3, 100, 0.3),            # the Fig. 9 shape
    (6000, 37, 0, 8, 100, 0.05), (6000, 37, 5, 110, 100, 0.02), (6000, 37, 0, 110, 7, 0.02),
    (4096, 128, 0, 17, 1, 0.01), (5000, 333, 30, 4, 4096, 0.2), (3000, 3000, 0, 110, 100, 0.0)])
def test_pec_s1_teacher_forced_bit_exact(L, N, W, cap, limit, big):
    tr = synth.trace(L, 777 + N)
    lat = synth.teacher_latencies(L, 55 + N, c_mean=30.0 if cap > 20 else 5.0, big=big)
    ref = oracle.simulate_pec(tr, N, W, limit=limit, forced_lat=lat, cap=cap)
    g = pec_run(tr, N, W, limit, cap=cap, forced=lat)
    _check_s1(g, ref)
    assert g["total"] == ref["total"]
    if N > 1 and limit > 0:
        assert ref["corr_len"].sum() > 0           # the case exercises the correction


@pytest.mark.parametrize("L,N,W,limit", [(6000, 60, 0, 100), (9001, 301, 20, 100), (4000, 40, 0, 3)])
def test_pec_s1_fused_kernels_forced_trajectory(L, N, W, limit):
    """PSIM_FORCE_PREDICT on bf16 C3 runs the fused conv_stack/fc1_head kernels (CNN
    evaluated every step) with the queue following the forced latencies: the fused
    update's stop rule and the step-0 block list of the correction pass are integer work."""
    tr = synth.trace(L, 91 + N)
    lat = synth.teacher_latencies(L, 17 + N, big=0.02)
    ref = oracle.simulate_pec(tr, N, W, limit=limit, forced_lat=lat)
    g = pec_run(tr, N, W, limit, forced=lat, weights=synth.weights("C3"), force_predict=True)
    assert np.array_equal(g["corr_len"], ref["corr_len"])
    assert np.array_equal(g["cycles1"], ref["cycles1"])
    assert np.array_equal(g["cycles"], ref["cycles"])
    assert np.array_equal(g["corr_k"], ref["corr_k"][g["first"]:])
    assert g["total"] == ref["total"]


@pytest.mark.parametrize("G", [2, 3])
def test_pec_rank_slices_first_subtrace_of_each_rank_not_corrected(G):
    L, N, W, limit = 8000, 90, 10, 100
    tr = synth.trace(L, 5)
    lat = synth.teacher_latencies(L, 6, big=0.03)
    ref = oracle.simulate_pec(tr, N, W, limit=limit, forced_lat=lat, G=G, want_rows=False)
    tot = 0
    for r in range(G):
        rr = P.partition_range(L, N, W, r, G)
        g = pec_run(tr[rr.row_lo:rr.row_hi], N, W, limit, forced=lat, rank=r, world=G, first_row=rr.row_lo,
                    n_instr=L, record=False)
        assert g["corr_len"][0] == 0
        assert np.array_equal(g["corr_len"], ref["corr_len"][rr.j0:rr.j1])
        assert np.array_equal(g["cycles"], ref["cycles"][rr.j0:rr.j1])
        tot += g["total"]
    assert tot == ref["total"]


def test_pec_off_and_single_subtrace():
    L = 3000
    tr = synth.trace(L, 8)
    lat = synth.teacher_latencies(L, 8, big=0.02)
    g = pec_run(tr, 1, 0, 100, forced=lat)
    assert g["corr_len"].tolist() == [0] and g["stats"]["corrected"] == 0
    assert g["total"] == oracle.simulate(tr, 1, 0, forced_lat=lat, want_rows=False)["total"]
    with P.Simulator(correction_limit=0) as sim:
        sim.load_trace(tr)
        sim.partition(4, 0)
        sim.force_latencies(lat)
        sim.simulate()
        with pytest.raises(P.PsimError):
            sim.corrections()
    with pytest.raises(P.PsimError):
        P.Simulator(correction_limit=100000)


@pytest.mark.parametrize("layerwise", [False, True])
def test_pec_s3_free_running_c3_bf16(layerwise):
    L, N, W, limit = 6000, 60, 0, 100
    tr = synth.trace(L, 2024)
    w = synth.weights("C3")
    ref = oracle.simulate_pec(tr, N, W, limit=limit, weights=w, mode=oracle.BF16, want_rows=False)
    g = pec_run(tr, N, W, limit, weights=w, layerwise=layerwise, record=False)
    assert abs(g["total"] - ref["total"]) <= 0.005 * ref["total"]
    assert abs(g["total"] - ref["total"]) < abs(ref["total1"] - ref["total"]) or ref["total1"] == ref["total"]
    assert abs(int(g["corr_len"].sum()) - int(ref["corr_len"].sum())) <= 0.1 * ref["corr_len"].sum() + 5
