"""Partitioning error trends on the GPU path (config 4 in miniature; PAPER.md:187-201,
Fig. 6): the error of the partitioned total against the same simulator at N = 1 grows
with N when there is no warm-up, and a warm-up of W >= Context_length rows
shrinks it.  The magnitudes are model-dependent (SURVEY §8c "partition error magnitude:
unpinned"); the test pins only the qualitative claims, with margins."""
import pytest

import paper_conf_sc_pandeylfhl22_b200 as P
import synth

pytestmark = pytest.mark.gpu


def total(tr, N, W, w):
    with P.Simulator(precision="bf16") as sim:
        sim.load_trace(tr)
        sim.partition(N, W)
        sim.load_model("C3", w)
        sim.simulate()
        return sim.total_cycles()


def test_partition_error_trends():
    L = 200_000
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 4)
    w = synth.weights("C3")
    ref = total(tr, 1, 0, w)
    err = {(N, W): (total(tr, N, W, w) - ref) / ref for N in (256, 4096, 16384) for W in (0, 128)}
    # no warm-up: cold boundaries cost cycles (queues start empty), more partitions, larger error
    assert abs(err[(256, 0)]) < abs(err[(4096, 0)]) < abs(err[(16384, 0)])
    assert abs(err[(16384, 0)]) > 0.05
    # warm-up of W >= Context_length: error back to the percent level at every N
    for N in (256, 4096, 16384):
        assert abs(err[(N, 128)]) < 0.03, err
        assert abs(err[(N, 128)]) < abs(err[(N, 0)]) or abs(err[(N, 0)]) < 0.01, err


def test_nccl_one_rank_communicator_leaves_results_unchanged():
    """The NCCL leg (one reduction at the end) executed for real: a 1-rank
    communicator built from psim_nccl_unique_id (the same call sequence a G-rank job
    uses) must give the same total and the same interval metrics as a run without a
    communicator (the fake-backend equivalent on one GPU).  NCCL cannot
    place two ranks on one device, so G > 1 is covered by the gloo host test and the
    emulated rank slices."""
    import numpy as np
    import synth
    L, N, W, I = 30_000, 96, 64, 500
    tr = synth.trace(L, 8181)
    w = synth.weights("C3")
    res = []
    for nid in (None, P.nccl_unique_id()):
        with P.Simulator(precision="bf16", interval=I, nccl_id=nid) as sim:
            sim.load_trace(tr)
            sim.partition(N, W)
            sim.load_model("C3", w)
            sim.simulate()
            res.append((sim.total_cycles(), sim.subtrace_cycles(), sim.interval_metrics(), sim.stats()["comm_ranks"]))
    (t0, c0, m0, r0), (t1, c1, m1, r1) = res
    assert r0 == 0 and r1 == 1
    assert t0 == t1 == int(c0.sum()) and np.array_equal(c0, c1)
    for k in ("cycles", "retired", "retired_st", "mem_bytes"):
        assert np.array_equal(m0[k], m1[k])


def test_long_unpartitioned_run_has_no_frozen_clock():
    """DESIGN.md R21 on the hot path over 1M unpartitioned rows of the config-4 trace (round
    1's model froze at row ~3.3M): the Clock never stands still for more than
    Context_length consecutive instructions, every completion latency is >= 1, and the
    statistics stay SPEC-like over the whole run (CPI, occupancy per 100k-row window)."""
    import numpy as np
    import synth
    L = 1_000_000
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 3)
    w = synth.weights("C3")
    with P.Simulator(precision="bf16", record_rows=True) as sim:
        sim.load_trace(tr)
        sim.partition(1, 0)
        sim.load_model("C3", w)
        sim.simulate()
        lat, k, clk = sim.get_rows(0, L)
    assert lat[:, 1].min() >= 1
    adv = np.diff(np.concatenate([[0], clk]))
    assert adv.min() >= 0
    runs = np.diff(np.concatenate([[-1], np.flatnonzero(adv != 0), [L]])) - 1   # zero-advance run lengths
    assert runs.max() <= 110, runs.max()
    for a in range(0, L, 100_000):
        cpi = (clk[a + 99_999] - (clk[a - 1] if a else 0)) / 100_000
        assert 0.5 < cpi < 4.0, (a, cpi)
        assert 5 < k[a:a + 100_000].mean() < 80, (a, k[a:a + 100_000].mean())
