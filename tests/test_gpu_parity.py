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
            record=True, rank=0, world=1, first_row=0, n_instr=None, device_trace=False, layerwise=False):
    with P.Simulator(precision=precision, queue_cap=cap, record_rows=record, rank=rank,
                     world_size=world, layerwise=layerwise) as sim:
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
    from test_oracle_queue import distinct_trace, parse_golden
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
    ref = oracle.simulate(tr, 1, 0, forced_lat=lat, cap=110)
    assert ref["clock"].max() > 2**32
    g = gpu_run(tr, 1, 0, forced=lat)
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
# DESIGN.md R17: the simulated dynamics are chaotic -- one legitimate rounding
# flip (fp32 summation order, R15) changes the context of every later
# instruction of that sub-trace, and the queue never drains to re-synchronise.
# So S3 is split: (a) decision agreement -- the GPU's gather + CNN + rounding on
# the ORACLE's trajectory (teacher-forced queue, PSIM_FORCE_PREDICT) must agree
# on >= 99.9% of per-instruction (f, c, s); (b) free-running totals within 0.5%.
def decision_parity(tr, N, arch, w, precision, samples=None, cap=110, layerwise=False):
    """W = 0 so the per-row forced latencies are exactly each sub-trace's oracle trajectory."""
    L = tr.shape[0]
    mode = oracle.BF16 if precision == "bf16" else oracle.FP64
    forced = synth.teacher_latencies(L, 17)
    rows = []
    js = range(N) if samples is None else samples
    for j in js:
        ref = oracle.simulate(tr, N, 0, arch=arch, weights=w, mode=mode, j0=j, nj=1, cap=cap)
        s, e = j * L // N, (j + 1) * L // N
        forced[s:e] = ref["lat"][s:e]
        rows.append((s, e))
    with P.Simulator(precision=precision, record_rows=True, force_predict=True, queue_cap=cap,
                     layerwise=layerwise) as sim:
        sim.load_trace(tr)
        sim.partition(N, 0)
        sim.load_model(arch, w)
        sim.force_latencies(forced)
        sim.simulate()
        agree, n = 0, 0
        for s, e in rows:
            lat, _, _ = sim.get_rows(s, e - s)
            agree += int(np.sum(np.all(lat == forced[s:e], axis=1)))
            n += e - s
    return agree / n


def free_running(tr, N, W, arch, w, precision, samples=None, layerwise=False):
    L = tr.shape[0]
    mode = oracle.BF16 if precision == "bf16" else oracle.FP64
    g = gpu_run(tr, N, W, arch=arch, weights=w, precision=precision, layerwise=layerwise)
    js = list(range(N)) if samples is None else list(samples)
    ref_c, gpu_c, agree, n = 0, 0, 0, 0
    for j in js:
        ref = oracle.simulate(tr, N, W, arch=arch, weights=w, mode=mode, j0=j, nj=1)
        s, e = j * L // N, (j + 1) * L // N
        ref_c += int(ref["cycles"][0]); gpu_c += int(g["cycles"][j])
        agree += int(np.sum(np.all(g["lat"][s:e] == ref["lat"][s:e], axis=1))); n += e - s
    return abs(gpu_c - ref_c) / ref_c, agree / n, g


def test_s3_config1_m2_fp32():
    """BASELINE.json configs[0]: 10k instructions, 1 sub-trace, queue 111, M2, fp32 --
    decision agreement and free-running total (N = 1, W = 0: both on the same run)."""
    L = 10_000
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 0)
    w = synth.weights("M2")
    assert decision_parity(tr, 1, "M2", w, "fp32") >= 0.999
    rel, agree, _ = free_running(tr, 1, 0, "M2", w, "fp32")
    assert rel <= 0.005


@pytest.mark.parametrize("precision,layerwise", [("bf16", False), ("bf16", True), ("fp32", False)])
def test_s3_c3_small(precision, layerwise):
    """bf16 runs the fused padding-aware kernels by default (layerwise=False) and the
    layer-by-layer tcgen05 GEMMs with layerwise=True; fp32 runs the SIMT path."""
    L, N = 3000, 6
    tr = synth.trace(L, 2024)
    w = synth.weights("C3")
    assert decision_parity(tr, N, "C3", w, precision, layerwise=layerwise) >= 0.999
    rel, agree, _ = free_running(tr, N, 64, "C3", w, precision, layerwise=layerwise)
    assert rel <= 0.005, (rel, agree)


def test_s3_fused_full_queue_and_ragged_tiles():
    """Fused path: contexts filled to the 110-entry cap (all 14 conv3 positions
    computed, P = 14) by long completion latencies, ragged sub-trace counts
    (N = 300: tiles of 128 + a partial tile) and finished sub-traces (ragged lengths)."""
    L, N = 45_017, 300                      # ~150 instructions per sub-trace, ragged
    tr = synth.trace(L, 99)
    w = synth.weights("C3")
    forced = synth.teacher_latencies(L, 23, c_mean=400.0)        # queues saturate: k -> 110, stalls
    mode = oracle.BF16
    refs = {}
    for j in (0, 7, 128, 255, 299):
        ref = oracle.simulate(tr, N, 0, forced_lat=forced, j0=j, nj=1, cap=110)
        refs[j] = ref
    # decision agreement of the CNN on those saturated trajectories
    with P.Simulator(precision="bf16", record_rows=True, force_predict=True) as sim:
        sim.load_trace(tr); sim.partition(N, 0); sim.load_model("C3", w); sim.force_latencies(forced)
        sim.simulate()
        st = sim.stats()
        assert max(i for i, c in enumerate(st["k_hist"]) if c) == 110
        agree, legit, n, bad = 0, 0, 0, []
        for j in refs:
            s, e = j * L // N, (j + 1) * L // N
            lat, k, clk = sim.get_rows(s, e - s)
            assert np.array_equal(k, refs[j]["k"][s:e]) and np.array_equal(clk, refs[j]["clock"][s:e])
            q = oracle.Queue(110)
            for i in range(s, e):            # the oracle's own CNN decision on the same state
                X, kk = q.build_input(tr, i)
                y = oracle.cnn_forward("C3", w, X, mode=mode)
                ref = tuple(oracle.round_latency(v) for v in y)
                got = tuple(int(v) for v in lat[i - s])
                n += 1
                if ref == got:
                    agree += 1
                elif all(r == g or abs(abs(v - np.floor(v)) - 0.5) <= 1e-3 * max(abs(v), 1.0)
                         for r, g, v in zip(ref, got, y)):
                    legit += 1                   # R15: within S2's tolerance of a .5 boundary
                else:
                    bad.append((i, kk, ref, got, y))
                q.update(i, *(int(v) for v in forced[i]))
        assert not bad and (agree + legit) / n >= 0.999 and agree / n >= 0.99, (agree, legit, n, bad[:5])


def test_s3_config2_full_size_sampled():
    """BASELINE.json configs[1] at full size (1M instructions, 1024 sub-traces, C3,
    bf16): decision agreement (W = 0) and free-running (W = 1000) on sampled
    sub-traces the oracle computes one by one."""
    L, N = 1_000_000, 1024
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 1)
    w = synth.weights("C3")
    assert decision_parity(tr, N, "C3", w, "bf16", samples=[0, 333, 517, 1023]) >= 0.999
    rel, agree, g = free_running(tr, N, 1000, "C3", w, "bf16", samples=[0, 201, 517, 640, 700, 967, 1023])
    assert rel <= 0.005, (rel, agree)
    assert g["stats"]["counted"] == L


@pytest.mark.slow
def test_s3_config3_full_size_sampled():
    """BASELINE.json configs[2] (100M instructions, 65536 sub-traces, bf16): the bench
    launch configuration, sampled sub-traces vs the oracle."""
    L, N = 100_000_000, 65536
    tr = synth.trace(L, synth.TRACE_SEED_BASE + 2)
    w = synth.weights("C3")
    assert decision_parity(tr, N, "C3", w, "bf16", samples=[0, 40000, 65535]) >= 0.999
    rel, agree, g = free_running(tr, N, 110, "C3", w, "bf16", samples=[0, 1, 9999, 32768, 40000, 65535])
    assert rel <= 0.005, (rel, agree)


@pytest.mark.parametrize("chunk", [0, 7])
def test_trace_residency_modes_identical(chunk):
    """The fused path gives bit-identical results whether the trace is resident in HBM,
    streamed from pinned host memory in chunks of lockstep steps (overlapped with the
    simulation), or staged from pageable memory."""
    L, N, W = 20_000, 64, 100
    tr = synth.trace(L, 4321)
    w = synth.weights("C3")
    totals, cycles = [], []
    pinned = torch.from_numpy(tr).pin_memory()
    for mode in ("device", "pinned", "pageable"):
        with P.Simulator(precision="bf16", chunk_steps=chunk) as sim:
            if mode == "device":
                sim.load_trace(torch.from_numpy(tr).cuda())
            elif mode == "pinned":
                sim.load_trace(pinned)
            else:
                sim.load_trace(tr)
            sim.partition(N, W)
            sim.load_model("C3", w)
            sim.simulate()
            totals.append(sim.total_cycles())
            cycles.append(sim.subtrace_cycles())
            st = sim.stats()
            assert st["trace_mode"] == {"device": 0, "pinned": 1, "pageable": 2}[mode]
    assert totals[0] == totals[1] == totals[2]
    assert np.array_equal(cycles[0], cycles[1]) and np.array_equal(cycles[0], cycles[2])


def test_fused_deterministic_many_tiles():
    """Race detector for the fused path: with several 128-block tiles per CTA per step
    (every pipeline buffer of conv_stack / fc1_head wraps many times), repeated runs and
    the pinned streaming mode give bit-identical per-sub-trace cycles.  (An early version
    of the conv3 staging buffer that a neighbouring warp could overwrite passed every
    single-tile test and failed exactly this.)"""
    L, N, W = 480_000, 40_000, 24
    tr = synth.trace(L, 777)
    w = synth.weights("C3")
    pinned = torch.from_numpy(tr).pin_memory()
    runs = []
    for src in ("device", "device", "pinned"):
        with P.Simulator(precision="bf16") as sim:
            sim.load_trace(torch.from_numpy(tr).cuda() if src == "device" else pinned)
            sim.partition(N, W)
            sim.load_model("C3", w)
            sim.simulate()
            runs.append((sim.total_cycles(), sim.subtrace_cycles()))
    for t, c in runs[1:]:
        assert t == runs[0][0] and np.array_equal(c, runs[0][1])
