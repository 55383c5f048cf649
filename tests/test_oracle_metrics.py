"""Pins of the oracle's interval metrics (PAPER.md:310-318 [VI-E]; R20).

"the simulator tracks the instruction retire events in the instruction queue
at a certain interval ... CPI ... the ratio of the collective predicted
instruction latency over the number of retired instructions for an interval";
stores are counted separately; memory bandwidth = data accessed from memory
(loads/stores whose data level is 2) over the latency.

Pins, none of which re-types oracle_simulate_metrics:
* the hand-traced 20-instruction table (tests/golden/hand_trace_cap4.txt):
  per-interval cycles from its clock columns and retire counts from its
  "retired" column;
* a brute-force retire-step computation from the retire-clock definition
  (PAPER.md:105-107): entry e retires in the first step t >= e whose Clock
  after the step is >= Clock_before(e) + f + c + s -- no queue, run per
  sub-trace on the clocks of a standalone N = 1 simulation of its rows
  (warm-up = simulating the W rows before it from an empty queue, R9);
* mem_bytes = a numpy bincount over the trace attributes (every row is
  counted by exactly one sub-trace, so it is independent of N and W);
* telescoping: sum of interval cycles = total cycles, for the CNN too.
"""
import numpy as np
import pytest

import oracle
import synth
from test_oracle_queue import distinct_trace, parse_golden


def golden_inputs():
    rows, _ = parse_golden()
    lat = np.array([r["lat"] for r in rows], np.uint16)
    tr = distinct_trace(20)
    stores = [3, 6, 9, 11, 13, 17]
    tr[stores, 8] = 1                                        # is_store
    tr[[2, 7, 13], 7] = 1                                    # is_load
    tr[[2, 7, 13, 17], 14] = [2, 2, 1, 2]                    # data level (13: L2, not memory)
    tr[[2, 7, 13, 17], 34] = [3, 6, 3, 2]                    # log2 access size
    return rows, lat, tr, set(stores)


@pytest.mark.parametrize("interval", [1, 3, 5, 7, 20, 64])
def test_metrics_hand_trace(interval):
    rows, lat, tr, stores = golden_inputs()
    m = oracle.simulate_metrics(tr, 1, 0, interval, forced_lat=lat, cap=4)
    ng = (20 + interval - 1) // interval
    cyc, ret, ret_st = np.zeros(ng, int), np.zeros(ng, int), np.zeros(ng, int)
    for r in rows:
        g = r["i"] // interval
        cyc[g] += r["clock_out"] - r["clock_in"]
        ret[g] += len(r["retired"])
        ret_st[g] += sum(1 for x, _ in r["retired"] if x in stores)
    assert m["cycles"].tolist() == cyc.tolist()
    assert m["retired"].tolist() == ret.tolist()
    assert m["retired_st"].tolist() == ret_st.tolist()
    mb = np.zeros(ng, int)
    mb[2 // interval] += 8
    mb[7 // interval] += 64
    mb[17 // interval] += 4                                  # a store served by memory counts too (:314)
    assert m["mem_bytes"].tolist() == mb.tolist()
    if interval == 5:
        # spelled out from the table: clocks 0->16->22->35->69, retires 2/5/6/6
        assert m["cycles"].tolist() == [16, 6, 13, 34]
        assert m["retired"].tolist() == [2, 5, 6, 6]


def brute_metrics(tr, lat, L, N, W, cap, interval):
    ng = (L + interval - 1) // interval
    cyc, ret, ret_st = (np.zeros(ng, np.int64) for _ in range(3))
    for j in range(N):
        s, e = j * L // N, (j + 1) * L // N
        ws = max(0, s - W)
        # the sub-trace alone: rows [ws, e) from an empty queue at Clock 0 (R9)
        sub = oracle.simulate(tr[ws:e], 1, 0, forced_lat=lat[ws:e], cap=cap)
        clk = sub["clock"]                                    # Clock after each row's step
        before = np.concatenate([[0], clk[:-1]])
        retire = before + lat[ws:e].astype(np.int64).sum(1)   # Clock_old + f + c + s
        for x in range(e - ws):
            t = x + int(np.argmax(clk[x:] >= retire[x])) if np.any(clk[x:] >= retire[x]) else None
            if t is None or ws + t < s:
                continue                                      # never retires / retires in warm-up
            g = (ws + t) // interval
            ret[g] += 1
            ret_st[g] += int(tr[ws + x, 8] != 0)
        for x in range(s - ws, e - ws):
            cyc[(ws + x) // interval] += clk[x] - before[x]
    return cyc, ret, ret_st


@pytest.mark.parametrize("N,W,cap,interval", [(1, 0, 110, 100), (1, 0, 6, 37), (7, 0, 8, 50),
                                              (7, 30, 8, 64), (13, 500, 110, 128), (5, 11, 3, 1)])
def test_metrics_brute_force(N, W, cap, interval):
    L = 1500
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 2)
    lat = synth.teacher_latencies(L, 11, f_mean=1.5, c_mean=25.0, s_mean=3.0, big=0.002)
    m = oracle.simulate_metrics(tr, N, W, interval, forced_lat=lat, cap=cap)
    cyc, ret, ret_st = brute_metrics(tr, lat, L, N, W, cap, interval)
    assert m["cycles"].tolist() == cyc.tolist()
    assert m["retired"].tolist() == ret.tolist()
    assert m["retired_st"].tolist() == ret_st.tolist()
    assert ret_st.sum() > 0 and ret.sum() > ret_st.sum()
    # mem bytes: plain definition over the trace attributes
    mem = ((tr[:, 7] | tr[:, 8]) != 0) & (tr[:, 14] == 2)
    mb = np.bincount(np.arange(L) // interval, weights=np.where(mem, 2.0 ** tr[:, 34], 0),
                     minlength=len(cyc)).astype(np.int64)
    assert m["mem_bytes"].tolist() == mb.tolist()
    # telescoping: interval cycles add up to the partitioned total
    assert int(m["cycles"].sum()) == oracle.simulate(tr, N, W, forced_lat=lat, cap=cap)["total"]


def test_metrics_unpartitioned_retire_count():
    # N = 1: everything fetched retires except what is still in the queue at the end
    L = 800
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 3)
    lat = synth.teacher_latencies(L, 5, c_mean=30.0)
    m = oracle.simulate_metrics(tr, 1, 0, 100, forced_lat=lat, cap=110)
    q = oracle.Queue(110)
    for i in range(L):
        q.update(i, *(int(v) for v in lat[i]))
    assert int(m["retired"].sum()) == L - len(q.entries())


def test_metrics_cnn_telescoping_and_identity():
    # the CNN path: interval cycles add up to the total; W >= s_j => partitioned
    # metrics equal unpartitioned metrics (identity ii of SURVEY §8c)
    L = 160
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 4)
    w = synth.weights("C3")
    m = oracle.simulate_metrics(tr, 4, 10, 16, arch="C3", weights=w)
    tot = oracle.simulate(tr, 4, 10, arch="C3", weights=w, want_rows=False)["total"]
    assert int(m["cycles"].sum()) == tot
    full = oracle.simulate_metrics(tr, 1, 0, 16, arch="C3", weights=w)
    part = oracle.simulate_metrics(tr, 4, L, 16, arch="C3", weights=w)
    for key in ("cycles", "retired", "retired_st", "mem_bytes"):
        assert part[key].tolist() == full[key].tolist(), key
    assert np.all(np.isfinite(full["cpi"][full["retired"] > 0]))


def test_metrics_bad_args():
    tr = synth.trace(50, synth.TRACE_SEED_BASE + 1)
    lat = synth.teacher_latencies(50, 1)
    with pytest.raises(ValueError):
        oracle.simulate_metrics(tr, 1, 0, 0, forced_lat=lat)
    with pytest.raises(ValueError):
        oracle.simulate_metrics(tr, 51, 0, 10, forced_lat=lat)
