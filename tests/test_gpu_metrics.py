"""GPU parity of the interval metrics (PAPER.md:310-318 [VI-E]; R20)
against oracle.simulate_metrics, through the C ABI (psim_opts.interval,
psim_get_interval_metrics).  Integer work: bit-exact.

* teacher-forced latencies on the warp update kernel (stalls, ragged
  intervals, N = L, W > s_j);
* the fused C3 kernels on the teacher-forced trajectory (PSIM_FORCE_PREDICT:
  gather + CNN run every step, the queue follows the forced latencies) with
  the trace resident, streamed from pinned memory and staged from pageable
  memory;
* G-rank slices: per-rank interval sums add up to the 1-rank metrics;
* the free-running bf16 C3 path: interval cycles add up to the total, memory
  bytes equal the trace's definition (independent of the trajectory);
* post-error correction on: metrics are the first pass's.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_pandeylfhl22_b200 as P
import synth

pytestmark = pytest.mark.gpu
KEYS = ("cycles", "retired", "retired_st", "mem_bytes")


def run(trace, N, W, interval, *, forced=None, weights=None, cap=110, force_predict=False, layerwise=False,
        mode="pageable", chunk=0, rank=0, world=1, first_row=0, n_instr=None, correction_limit=0):
    with P.Simulator(precision="bf16", queue_cap=cap, force_predict=force_predict, layerwise=layerwise,
                     interval=interval, chunk_steps=chunk, rank=rank, world_size=world,
                     correction_limit=correction_limit) as sim:
        if mode == "device":
            sim.load_trace(torch.from_numpy(np.ascontiguousarray(trace)).cuda(), n_instr=n_instr, first_row=first_row)
        elif mode == "pinned":
            sim.load_trace(torch.from_numpy(np.ascontiguousarray(trace)).pin_memory(), n_instr=n_instr,
                           first_row=first_row)
        else:
            sim.load_trace(trace, n_instr=n_instr, first_row=first_row)
        sim.partition(N, W)
        if weights is not None:
            sim.load_model("C3", weights)
        if forced is not None:
            sim.force_latencies(forced)
        sim.simulate()
        return sim.interval_metrics(), sim.total_cycles()


def check(m, ref):
    for k in KEYS:
        assert np.array_equal(m[k], ref[k]), (k, np.nonzero(m[k] != ref[k])[0][:10])


@pytest.mark.parametrize("L,N,W,cap,interval,big", [
    (6000, 1, 0, 110, 1000, 0.0), (6000, 37, 50, 8, 64, 0.02), (3000, 3000, 3, 110, 7, 0.0),
    (5000, 333, 1000, 1, 100, 0.0), (7919, 64, 110, 110, 1, 0.05), (4096, 128, 0, 17, 4096, 0.01)])
def test_metrics_teacher_forced_bit_exact(L, N, W, cap, interval, big):
    tr = synth.trace(L, 4242 + N)
    lat = synth.teacher_latencies(L, 99 + N, c_mean=30.0 if cap > 20 else 5.0, big=big)
    ref = oracle.simulate_metrics(tr, N, W, interval, forced_lat=lat, cap=cap)
    m, total = run(tr, N, W, interval, forced=lat, cap=cap)
    check(m, ref)
    assert int(m["cycles"].sum()) == total
    assert m["retired_st"].sum() > 0


@pytest.mark.parametrize("mode,chunk", [("device", 0), ("pinned", 0), ("pinned", 5), ("pageable", 0)])
def test_metrics_fused_forced_trajectory(mode, chunk):
    L, N, W, interval = 12_000, 200, 60, 250
    tr = synth.trace(L, 777)
    lat = synth.teacher_latencies(L, 8, c_mean=30.0, big=0.01)
    ref = oracle.simulate_metrics(tr, N, W, interval, forced_lat=lat, cap=110)
    m, _ = run(tr, N, W, interval, forced=lat, weights=synth.weights("C3"), force_predict=True, mode=mode,
               chunk=chunk)
    check(m, ref)


def test_metrics_layerwise_forced_trajectory():
    L, N, W, interval = 4000, 50, 30, 33
    tr = synth.trace(L, 778)
    lat = synth.teacher_latencies(L, 9, c_mean=30.0)
    ref = oracle.simulate_metrics(tr, N, W, interval, forced_lat=lat, cap=110)
    m, _ = run(tr, N, W, interval, forced=lat, weights=synth.weights("C3"), force_predict=True, layerwise=True)
    check(m, ref)


def test_metrics_rank_slices_sum():
    L, N, W, interval = 9000, 101, 77, 300
    tr = synth.trace(L, 31)
    lat = synth.teacher_latencies(L, 3, big=0.01)
    ref = oracle.simulate_metrics(tr, N, W, interval, forced_lat=lat, cap=110)
    for G in (2, 3):
        acc = {k: np.zeros_like(ref[k]) for k in KEYS}
        for r in range(G):
            rr = P.partition_range(L, N, W, r, G)
            m, _ = run(tr[rr.row_lo:rr.row_hi], N, W, interval, forced=lat, rank=r, world=G, first_row=rr.row_lo,
                       n_instr=L)
            for k in KEYS:
                acc[k] += m[k]
        check(acc, ref)


def test_metrics_free_running_c3():
    L, N, W, interval = 30_000, 64, 110, 1000
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 2)
    w = synth.weights("C3")
    m, total = run(tr, N, W, interval, weights=w)
    assert int(m["cycles"].sum()) == total
    mem = ((tr[:, 7] | tr[:, 8]) != 0) & (tr[:, 14] == 2)
    mb = np.bincount(np.arange(L) // interval, weights=np.where(mem, 2.0 ** tr[:, 34], 0)).astype(np.int64)
    assert np.array_equal(m["mem_bytes"], mb)
    ref = oracle.simulate_metrics(tr, N, W, interval, arch="C3", weights=w, mode=oracle.BF16)
    # trajectories may legitimately diverge after a rounding flip (R17): aggregate CPI within 0.5%
    cpi_g = m["cycles"].sum() / m["retired"].sum()
    cpi_o = ref["cycles"].sum() / ref["retired"].sum()
    assert abs(cpi_g - cpi_o) / cpi_o <= 0.005


def test_metrics_with_correction_are_first_pass():
    L, N, W, interval = 6000, 40, 0, 500
    tr = synth.trace(L, 55)
    lat = synth.teacher_latencies(L, 4, c_mean=30.0)
    ref = oracle.simulate_metrics(tr, N, W, interval, forced_lat=lat, cap=110)
    m, _ = run(tr, N, W, interval, forced=lat, correction_limit=100)
    check(m, ref)


def test_metrics_errors():
    tr = synth.trace(100, 1)
    with P.Simulator() as sim:
        sim.load_trace(tr)
        sim.partition(2, 0)
        sim.force_latencies(synth.teacher_latencies(100, 1))
        sim.simulate()
        with pytest.raises(P.PsimError) as e:
            sim.interval_metrics(0, 1)
        assert e.value.code == P.ERR_STATE
    with pytest.raises(P.PsimError):
        P.Simulator(interval=P.MAX_INTERVAL + 1)
    with P.Simulator(interval=10) as sim:
        sim.load_trace(tr)
        sim.partition(2, 0)
        sim.force_latencies(synth.teacher_latencies(100, 1))
        sim.simulate()
        with pytest.raises(P.PsimError) as e:
            sim.interval_metrics(5, 6)
        assert e.value.code == P.ERR_ARG
        assert len(sim.interval_metrics()["cycles"]) == 10
