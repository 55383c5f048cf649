"""GPU parity: the CUDA path through the C ABI vs the CPU oracle (stages S1-S3,
DESIGN.md "parity"), element by element on the same seeded inputs.

S1  teacher-forced latencies: context counts, Clocks, boundary, per-sub-trace
    cycles and totals bit-exact (integer work).
S2  CNN forward on fixed inputs: max|dy| / max(|y_ref|, 1) <= 1e-3 (fp32 path
    vs fp64 oracle) and <= 2e-2 (bf16 path vs fp64 oracle; BASELINE.json
    north_star); bf16 path vs the bf16-operand oracle <= 1e-3 (same rounding
    points, different fp32 summation order -- DESIGN.md R16).
S3  end to end, same N and W: >= 99.9% of per-instruction (f, c, s) agree and
    total cycles within 0.5% (north_star), bf16 GPU vs bf16 oracle and fp32 GPU
    vs fp64 oracle.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_pandeylfhl22_b200 as P
import synth

pytestmark = pytest.mark.gpu


def gpu_run(trace, N, W, *, arch="C3", weights=None, precision="bf16", cap=110, forced=None,
            record=True, rank=0, world=1, first_row=0, n_instr=None, device_trace=False):
    with P.Simulator(precision=precision, queue_cap=cap, record_rows=record, rank=rank,
                     world_size=world) as sim:
        if device_trace:
            t = torch.from_numpy(np.ascontiguousarray(trace)).cuda()
            sim.load_trace(t, n_instr=n_instr, first_row=first_row)
        else:
            sim.load_trace(trace, n_instr=n_instr, first_row=first_row)
        sim.partition(N, W)
        if forced is not None:
            sim.force_latencies(forced)
        else:
            sim.load_model(arch, weights)
        sim.simulate()
        rr = sim.rank_range()
        out = dict(total=sim.total_cycles(), cycles=sim.subtrace_cycles(), stats=sim.stats(), rr=rr)
        if record and rr.j1 > rr.j0:
            L = n_instr if n_instr is not None else trace.shape[0]
            s0 = rr.j0 * L // N
            lat, k, clk = sim.get_rows(s0, rr.row_hi - s0)
            out.update(lat=lat, k=k, clock=clk, first=s0)
        return out


# ------------------------------------------------------------------ S1
def test_s1_hand_trace_partitions():
    from tests.test_oracle_queue import distinct_trace, parse_golden
    rows, parts = parse_golden()
    lat = np.array([r["lat"] for r in rows], np.uint16)
    tr = distinct_trace(20)
    for W, cyc, total in parts:
        g = gpu_run(tr, 4, W, cap=4, forced=lat)
        assert g["cycles"].tolist() == cyc and g["total"] == total
    g = gpu_run(tr, 1, 0, cap=4, forced=lat)
    assert g["total"] == 69
    assert g["clock"].tolist() == [r["clock_out"] for r in rows]
    assert g["k"].tolist() == [len(r["ctx"]) for r in rows]


@pytest.mark.parametrize("L,N,W,cap,big", [
    (6000, 1, 0, 110, 0.0), (6000, 37, 50, 8, 0.02), (6000, 6000, 3, 110, 0.0),
    (5000, 333, 1000, 1, 0.0), (7919, 64, 110, 110, 0.05), (4096, 128, 0, 17, 0.01)])
def test_s1_teacher_forced_bit_exact(L, N, W, cap, big):
    tr = synth.trace(L, 4242 + N)
    lat = synth.teacher_latencies(L, 99 + N, c_mean=30.0 if cap > 20 else 5.0, big=big)
    ref = oracle.simulate(tr, N, W, forced_lat=lat, cap=cap)
    g = gpu_run(tr, N, W, cap=cap, forced=lat)
    assert np.array_equal(g["k"], ref["k"])
    assert np.array_equal(g["clock"], ref["clock"])
    assert np.array_equal(g["cycles"], ref["cycles"])
    assert g["total"] == ref["total"]
    assert g["stats"]["stalls"] == ref["stalls"]


def test_s1_clock_beyond_32_bits():
    # fetch latencies at the clamp (4095) push the Clock past 2^32: the low-32-bit
    # age arithmetic must stay exact.
    L = 1_100_000
    tr = np.zeros((L, 48), np.uint8)
    lat = synth.teacher_latencies(L, 5, c_mean=30.0)
    lat[:, 0] = 4095
    ref = oracle.simulate(tr, 2, 10, forced_lat=lat, cap=110)
    assert ref["clock"].max() > 2**32
    g = gpu_run(tr, 2, 10, forced=lat)
    assert np.array_equal(g["clock"], ref["clock"]) and np.array_equal(g["k"], ref["k"])
    assert g["total"] == ref["total"]


def test_s1_device_resident_trace_and_rank_slices():
    """Inputs resident in HBM give the same result; G ranks on their own row slices
    sum (int64) to the 1-rank total bit-exactly (sub-traces are independent)."""
    L, N, W = 9000, 101, 77
    tr = synth.trace(L, 31)
    lat = synth.teacher_latencies(L, 3, big=0.01)
    ref = oracle.simulate(tr, N, W, forced_lat=lat, cap=110, want_rows=False)
    g1 = gpu_run(tr, N, W, forced=lat, device_trace=True)
    assert g1["total"] == ref["total"]
    for G in (2, 3, 8):
        tot = 0
        for r in range(G):
            rr = P.partition_range(L, N, W, r, G)
            gr = gpu_run(tr[rr.row_lo:rr.row_hi], N, W, forced=lat, rank=r, world=G, first_row=rr.row_lo,
                         n_instr=L, record=False)
            assert np.array_equal(gr["cycles"], ref["cycles"][rr.j0:rr.j1])
            tot += gr["total"]
        assert tot == ref["total"]


def test_state_machine_and_argument_errors():
    tr = synth.trace(100, 1)
    with P.Simulator() as sim:
        with pytest.raises(P.PsimError) as e:
            sim.simulate()
        assert e.value.code == P.ERR_STATE
        with pytest.raises(P.PsimError):
            sim.total_cycles()
        sim.load_trace(tr)
        with pytest.raises(P.PsimError) as e:
            sim.partition(101, 0)
        assert e.value.code == P.ERR_ARG
        sim.partition(10, 5)
        with pytest.raises(P.PsimError) as e:
            sim.load_model("C3", synth.weights("C3")[:-1])
        assert e.value.code == P.ERR_ARG
        with pytest.raises(P.PsimError) as e:
            sim.simulate()                       # no model, no forcing
        assert e.value.code == P.ERR_STATE
        with pytest.raises(P.PsimError) as e:
            sim.load_trace(tr[:, :40])           # stride < 48
        assert e.value.code == P.ERR_ARG


# ------------------------------------------------------------------ S2
def s2_inputs(n, seed):
    """Gathered inputs from a teacher-forced oracle run: k from 0 to 110 (long
    completions fill the queue), plus adversarial time values."""
    tr = synth.trace(3000, 777 + seed)
    lat = synth.teacher_latencies(3000, seed, c_mean=20.0)
    lat[1000:1200, 1] = 4000                       # fill the queue to 110
    q = oracle.Queue(110)
    Xs, ks = [], []
    for i in range(3000):
        X, k = q.build_input(tr, i)
        if i % (3000 // n) == 0 or k == 110 and len([x for x in ks if x == 110]) < 3:
            Xs.append(X); ks.append(k)
        q.update(i, *(int(v) for v in lat[i]))
    rng = np.random.default_rng(seed)
    for _ in range(8):
        X = Xs[rng.integers(len(Xs))].copy()
        X[:, :3] = np.where(X[:, 3:4] > 0, rng.integers(0, 8191, (112, 3)), 0)
        Xs.append(X); ks.append(-1)
    assert 0 in ks and 110 in ks
    return np.stack(Xs)


def s2_err(y, ref):
    return float(np.max(np.abs(y - ref)) / max(float(np.max(np.abs(ref))), 1.0))


@pytest.mark.parametrize("arch", ["M2", "C3"])
def test_s2_cnn_fp32(arch):
    w = synth.weights(arch)
    X = s2_inputs(300, 1)
    with P.Simulator(precision="fp32") as sim:
        sim.load_model(arch, w)
        y = sim.cnn_forward(X)
    ref = np.stack([oracle.cnn_forward(arch, w, x) for x in X])
    assert s2_err(y, ref) <= 1e-3


@pytest.mark.parametrize("arch", ["M2", "C3"])
def test_s2_cnn_bf16_tensor_cores(arch):
    w = synth.weights(arch)
    X = s2_inputs(300, 2)
    with P.Simulator(precision="bf16") as sim:
        sim.load_model(arch, w)
        y = sim.cnn_forward(X)
    ref64 = np.stack([oracle.cnn_forward(arch, w, x) for x in X])
    ref16 = np.stack([oracle.cnn_forward(arch, w, x, mode=oracle.BF16) for x in X])
    assert s2_err(y, ref64) <= 2e-2
    assert s2_err(y, ref16) <= 1e-3


# ------------------------------------------------------------------ S3
def s3_check(g, ref, L):
    real = ref["k"] >= 0
    lat_g = g["lat"][real[g["first"]:]] if g["first"] else g["lat"][real]
    agree = np.mean(np.all(lat_g == ref["lat"][real], axis=1))
    rel = abs(g["total"] - ref["total"]) / max(ref["total"], 1)
    return agree, rel


def test_s3_config1_m2_fp32():
    """BASELINE.json configs[0]: 10k instructions, 1 sub-trace, queue 111, M2, fp32."""
    L = 10_000
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 0)
    w = synth.weights("M2")
    ref = oracle.simulate(tr, 1, 0, arch="M2", weights=w)
    g = gpu_run(tr, 1, 0, arch="M2", weights=w, precision="fp32")
    agree, rel = s3_check(g, ref, L)
    assert agree >= 0.999 and rel <= 0.005, (agree, rel)


def test_s3_c3_bf16_partitioned():
    L, N, W = 2500, 8, 64
    tr = synth.trace(L, 2024)
    w = synth.weights("C3")
    ref = oracle.simulate(tr, N, W, arch="C3", weights=w, mode=oracle.BF16)
    g = gpu_run(tr, N, W, arch="C3", weights=w, precision="bf16")
    agree, rel = s3_check(g, ref, L)
    assert agree >= 0.999 and rel <= 0.005, (agree, rel)
    assert np.all(np.abs(g["cycles"] - ref["cycles"]) <= np.maximum(0.005 * ref["cycles"], 2))


def test_s3_c3_fp32_partitioned():
    L, N, W = 1500, 5, 40
    tr = synth.trace(L, 2025)
    w = synth.weights("C3")
    ref = oracle.simulate(tr, N, W, arch="C3", weights=w)
    g = gpu_run(tr, N, W, arch="C3", weights=w, precision="fp32")
    agree, rel = s3_check(g, ref, L)
    assert agree >= 0.999 and rel <= 0.005, (agree, rel)


def sampled_parity(L, N, W, seed, samples, precision="bf16"):
    tr = synth.trace(L, seed)
    w = synth.weights("C3")
    with P.Simulator(precision=precision, record_rows=True) as sim:
        sim.load_trace(tr)
        sim.partition(N, W)
        sim.load_model("C3", w)
        sim.simulate()
        cyc = sim.subtrace_cycles()
        agree, n_rows = 0, 0
        for j in samples:
            ref = oracle.simulate(tr, N, W, arch="C3", weights=w, j0=j, nj=1,
                                  mode=oracle.BF16 if precision == "bf16" else oracle.FP64)
            s, e = j * L // N, (j + 1) * L // N
            lat, k, clk = sim.get_rows(s, e - s)
            agree += int(np.sum(np.all(lat == ref["lat"][s:e], axis=1)))
            n_rows += e - s
            assert abs(int(cyc[j]) - int(ref["cycles"][0])) <= max(0.005 * ref["cycles"][0], 2), j
        return agree / n_rows, sim.stats()


def test_s3_config2_sampled():
    """BASELINE.json configs[1] at full size (1M instructions, 1024 sub-traces,
    W = 1000, C3, bf16) on sampled sub-traces the oracle computes one by one."""
    agree, st = sampled_parity(1_000_000, 1024, 1000, synth.TRACE_SEED_BASE + 1, [0, 517, 1023])
    assert agree >= 0.999
    assert st["counted"] == 1_000_000


@pytest.mark.slow
def test_s3_config3_sampled():
    """BASELINE.json configs[2] (100M instructions, 65536 sub-traces, bf16) in the
    bench launch configuration, sampled sub-traces vs the oracle."""
    agree, st = sampled_parity(100_000_000, 65536, 110, synth.TRACE_SEED_BASE + 2, [0, 40000, 65535])
    assert agree >= 0.999
    assert st["counted"] == 100_000_000
