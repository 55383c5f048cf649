"""Pins of the oracle's queue / clock / retire rules (Fig. 1).

Pins, none of which re-types the oracle's own code:
* the numbers the paper prints for Fig. 1;
* a hand-traced 20-instruction table (tests/golden/hand_trace_cap4.txt);
* a brute-force simulator written from the *set* definition of the context
  ("the instruction queue holds all the instructions currently executing",
  PAPER.md:91): context of i = {j < i : retire_j > Clock}, scanned over all
  previous instructions with no queue at all;
* closed forms: context-free latencies without overflow => total = sum f;
* invariants I1-I4 (clock monotone, |Q| <= cap, retire order non-decreasing,
  every live entry has retire > Clock).
"""
import os
import re

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hand_trace_cap4.txt")


def parse_golden():
    rows, parts = [], []
    for line in open(GOLD):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        if line.startswith("partition"):
            m = re.match(r"partition W=(\d+) \| ([\d ]+) \| (\d+)", line)
            parts.append((int(m.group(1)), [int(x) for x in m.group(2).split()], int(m.group(3))))
            continue
        f = [x.strip() for x in line.split("|")]
        i = int(f[0])
        lat = tuple(int(x) for x in f[1].split())
        ctx = [] if f[3] == "-" else [
            (int(m.group(1)), (int(m.group(2)), int(m.group(3)), int(m.group(4))))
            for m in re.finditer(r"(\d+):\((\d+),(\d+),(\d+)\)", f[3])]
        ret = [] if f[6] == "-" else [tuple(int(y) for y in x.split("@")) for x in f[6].split()]
        q = [tuple(int(y) for y in x.split("@")) for x in f[7].split()]
        rows.append(dict(i=i, lat=lat, clock_in=int(f[2]), ctx=ctx, clock_out=int(f[4]),
                         stall=int(f[5]), retired=ret, queue=q))
    return rows, parts


def distinct_trace(L):
    """Rows whose attribute bytes identify the instruction (attr0 = i, attr1 = i>>8)."""
    tr = np.zeros((L, 48), np.uint8)
    tr[:, 0] = np.arange(L) & 0xFF
    tr[:, 1] = np.arange(L) >> 8
    tr[:, 2] = 7
    return tr


def test_paper_fig1_numbers():
    # first instruction predicts 13, 1, 0; Clock 0 + 13 = 13;
    # retire clock 13 + 1 + 0 = 14.  PAPER.md:107: at Clock 15 (iteration 2) it
    # retires and is no longer context.
    tr = distinct_trace(3)
    q = oracle.Queue(cap=2)            # input length 3 = Context_length + 1
    X, k = q.build_input(tr, 0)
    assert k == 0 and np.all(X[1:] == 0) and X[0, 3] == 0 and X[0, 5] == 7
    retired, stall = q.update(0, 13, 1, 0)
    assert q.clock == 13 and not stall and retired == []
    (seq, fetch, complete, retire), = q.entries()
    assert (seq, retire) == (0, 14)
    X, k = q.build_input(tr, 1)
    assert k == 1 and X[1, 3] == 0                  # instruction 0 is context of instruction 1
    retired, _ = q.update(1, 2, 3, 0)               # Clock 13 -> 15
    assert q.clock == 15 and retired == [(0, 14)]   # 15 >= 14: retires
    X, k = q.build_input(tr, 2)
    assert k == 1 and X[1, 3] == 1                  # only instruction 1 remains


def test_hand_trace_table():
    rows, _ = parse_golden()
    tr = distinct_trace(20)
    q = oracle.Queue(cap=4)
    for r in rows:
        assert q.clock == r["clock_in"], r["i"]
        X, k = q.build_input(tr, r["i"])
        assert k == len(r["ctx"])
        assert X[0, 3] == r["i"] and tuple(X[0, :3]) == (0, 0, 0)   # current first, no time
        for row, (seq, tf) in enumerate(r["ctx"], 1):
            assert X[row, 3] == seq, (r["i"], row)
            assert tuple(int(v) for v in X[row, :3]) == tf, (r["i"], row)
        assert np.all(X[k + 1:] == 0)                                 # zero padding at the tail
        retired, stall = q.update(r["i"], *r["lat"])
        assert q.clock == r["clock_out"], r["i"]
        assert int(stall) == (1 if r["stall"] else 0)
        assert sorted(retired) == sorted(r["retired"]), r["i"]
        assert [(e[0], e[3]) for e in q.entries()] == r["queue"], r["i"]
    assert q.clock == 69 and q.stalls == 2


def test_hand_trace_partitions():
    rows, parts = parse_golden()
    lat = np.array([r["lat"] for r in rows], np.uint16)
    tr = distinct_trace(20)
    for W, cyc, total in parts:
        out = oracle.simulate(tr, 4, W, forced_lat=lat, cap=4)
        assert out["cycles"].tolist() == cyc, W
        assert out["total"] == total
    # unpartitioned (N=1) total = final clock of the table
    assert oracle.simulate(tr, 1, 0, forced_lat=lat, cap=4)["total"] == 69
    # capacity 110: no stall, total = sum f for every W (closed form)
    for W in (0, 3, 5, 20):
        assert oracle.simulate(tr, 4, W, forced_lat=lat, cap=110)["total"] == int(lat[:, 0].sum())


# ---------------------------------------------------------------------------
# brute force from the set definition (no queue)
# ---------------------------------------------------------------------------
def brute_force(lat, L, N, W, cap):
    """Per sub-trace: clock chain by scanning all earlier instructions."""
    out_k = np.full(L, -1, np.int64)
    out_clock = np.zeros(L, np.int64)
    out_ctx = {}
    cycles = []
    for j in range(N):
        s, e = j * L // N, (j + 1) * L // N
        ws = max(0, s - W)
        clock, bnd = 0, 0
        retire = {}
        for i in range(ws, e):
            live = sorted((x for x in retire if retire[x] > clock), reverse=True)
            if i >= s:
                out_k[i] = len(live)
                out_ctx[i] = live
            f, c, st = (int(v) for v in lat[i])
            clock += f
            retire[i] = clock + c + st
            alive = [x for x in retire if retire[x] > clock]
            if len(alive) > cap:
                clock = min(retire[x] for x in alive)
            if i == s - 1:
                bnd = clock
            if i >= s:
                out_clock[i] = clock
        cycles.append(clock - bnd)
    return out_k, out_clock, np.array(cycles), out_ctx


@pytest.mark.parametrize("seed,cap,N,W,big", [
    (1, 3, 1, 0, 0.0), (2, 4, 3, 2, 0.0), (3, 8, 5, 7, 0.02), (4, 110, 4, 50, 0.01),
    (5, 16, 7, 0, 0.05), (6, 2, 2, 300, 0.0)])
def test_bruteforce_agreement(seed, cap, N, W, big):
    L = 400
    lat = synth.teacher_latencies(L, seed, c_mean=6.0 if cap < 20 else 20.0, big=big)
    tr = distinct_trace(L)
    out = oracle.simulate(tr, N, W, forced_lat=lat, cap=cap)
    k, clk, cyc, ctx = brute_force(lat, L, N, W, cap)
    assert np.array_equal(out["k"], k)
    assert np.array_equal(out["clock"], clk)
    assert np.array_equal(out["cycles"], cyc)
    # context identity and ordering (newest first) for sub-trace 0 via the queue API
    q = oracle.Queue(cap)
    e0 = L // N
    for i in range(e0):
        X, kk = q.build_input(tr, i)
        seqs = [int(X[r, 3]) + 256 * int(X[r, 4]) for r in range(1, kk + 1)]
        assert seqs == ctx[i]
        q.update(i, *(int(v) for v in lat[i]))


def test_invariants_random():
    L, cap = 3000, 12
    lat = synth.teacher_latencies(L, 11, c_mean=8.0, s_mean=3.0, big=0.01)
    tr = distinct_trace(L)
    q = oracle.Queue(cap)
    prev_clock = 0
    retire_seq = []
    for i in range(L):
        _, k = q.build_input(tr, i)
        assert k <= cap                                    # I2
        retired, _ = q.update(i, *(int(v) for v in lat[i]))
        retire_seq += sorted(r for _, r in retired)
        assert q.clock >= prev_clock                       # I1
        prev_clock = q.clock
        assert all(e[3] > q.clock for e in q.entries())    # I4
        assert len(q.entries()) <= cap
    assert all(a <= b for a, b in zip(retire_seq, retire_seq[1:]))   # I3
    assert q.stalls > 0                                    # the case was exercised


def test_context_free_closed_form():
    # no overflow (cap 110, short latencies): total == sum of fetch latencies for any N, W
    L = 2000
    lat = synth.teacher_latencies(L, 21, f_mean=2.0, c_mean=3.0, s_mean=1.0)
    tr = distinct_trace(L)
    for N, W in [(1, 0), (7, 0), (13, 40), (250, 1000), (L, 3)]:
        out = oracle.simulate(tr, N, W, forced_lat=lat, cap=110)
        assert out["stalls"] == 0
        assert out["total"] == int(lat[:, 0].astype(np.int64).sum()), (N, W)


def test_rounding_special_cases():
    rl = oracle.round_latency
    assert [rl(v) for v in (0.5, 1.5, 2.5, -0.3, -7.0, 0.49999997, 3.5000002)] == [0, 2, 2, 0, 0, 0, 4]
    assert rl(4095.6) == 4095 and rl(1e10) == 4095 and rl(float("inf")) == 4095
    assert rl(float("nan")) == 0 and rl(float("-inf")) == 0
    assert rl(4094.5) == 4094 and rl(4093.5) == 4094
