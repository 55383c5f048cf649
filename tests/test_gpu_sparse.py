"""GPU parity of the 2:4 structured-sparse path (PSIM_SPARSE24: tcgen05.mma.sp on every
tensor-core layer, gemm_sp.cu; PAPER.md:157 [IV-B], :261 [VI-B]) against the oracle on the
same 2:4-pruned weights (R22), through the C ABI.

S2: CNN forward on fixed gathered inputs (k = 0 .. 110 and adversarial times): <= 2e-2 vs the
    fp64 oracle, vs the bf16-operand oracle the bf16 bound of test_gpu_parity (worst row 5e-3,
    median 1e-5) -- the sparse MMA computes the same products as the dense one.
S3: decision agreement on the oracle's trajectory (every disagreement a rounding-boundary
    case, R15) and free-running totals within 0.5%, sparse C3 and sparse M2.
The sparse and the dense layer-wise GEMMs on the same pruned weights agree to fp32 noise, and
a model that is not 2:4 sparse is rejected (ARG)."""
import numpy as np
import pytest

import oracle
import paper_conf_sc_pandeylfhl22_b200 as P
import synth
from test_gpu_parity import Y_MEDIAN, Y_TOL, _legit_flip, s2_inputs

pytestmark = pytest.mark.gpu


def _rows_err(y, ref):
    return np.max(np.abs(y - ref), axis=1) / np.maximum(np.max(np.abs(ref), axis=1), 1.0)


@pytest.mark.parametrize("arch", ["C3", "M2"])
def test_s2_sparse_cnn(arch):
    w = synth.weights(arch, sparse24=True)
    X = s2_inputs(300, 7)
    with P.Simulator(precision="bf16", sparse24=True) as sim:
        sim.load_model(arch, w)
        y = sim.cnn_forward(X)
    with P.Simulator(precision="bf16", layerwise=True) as sim:      # dense tcgen05 GEMMs, same weights
        sim.load_model(arch, w)
        y_dense = sim.cnn_forward(X)
    ref64 = np.stack([oracle.cnn_forward(arch, w, x) for x in X])
    ref16 = np.stack([oracle.cnn_forward(arch, w, x, mode=oracle.BF16) for x in X])
    e64, e16, ed = _rows_err(y, ref64), _rows_err(y, ref16), _rows_err(y, y_dense)
    print(f"S2 sparse {arch}: vs fp64 max {e64.max():.2e}; vs bf16 max {e16.max():.2e} median {np.median(e16):.2e}; "
          f"vs dense GEMM max {ed.max():.2e}")
    if arch == "C3":
        # north_star bf16 bound vs the exact CNN.  (The pruned M2 -- config 1's model is dense fp32;
        # a bf16 2:4 M2 is not a configured workload -- amplifies bf16 operand rounding to ~1e-1
        # against fp64 in the bf16-operand ORACLE as well, so only the same-precision bound below
        # applies to it.)
        assert e64.max() <= 2e-2
    assert e16.max() <= Y_TOL["bf16"] and np.median(e16) <= Y_MEDIAN
    assert ed.max() <= Y_TOL["bf16"] and np.median(ed) <= Y_MEDIAN


def test_dense_model_rejected_by_sparse_path():
    with P.Simulator(precision="bf16", sparse24=True) as sim:
        with pytest.raises(P.PsimError) as e:
            sim.load_model("C3", synth.weights("C3"))
        assert e.value.code == P.ERR_ARG
    with P.Simulator(precision="fp32", sparse24=True) as sim:
        with pytest.raises(P.PsimError) as e:
            sim.load_model("C3", synth.weights("C3", sparse24=True))
        assert e.value.code == P.ERR_UNSUPPORTED


@pytest.mark.parametrize("arch,L,N", [("C3", 3000, 6), ("M2", 2000, 4), ("C3", 40_000, 300)])
def test_s3_sparse(arch, L, N):
    """Decision agreement (W = 0, oracle trajectory) on all sub-traces of the small cases,
    sampled on the ragged 300-sub-trace case (several 128-row GEMM tiles per layer);
    free-running totals within 0.5%."""
    tr = synth.trace(L, 3131 + N)
    w = synth.weights(arch, sparse24=True)
    samples = None if N <= 8 else [0, 127, 128, 299]
    forced = synth.teacher_latencies(L, 17)
    ref_y = np.zeros((L, 3), np.float32)
    rows = []
    for j in (range(N) if samples is None else samples):
        ref = oracle.simulate(tr, N, 0, arch=arch, weights=w, mode=oracle.BF16, j0=j, nj=1)
        s, e = j * L // N, (j + 1) * L // N
        forced[s:e] = ref["lat"][s:e]
        ref_y[s:e] = ref["y"][s:e]
        rows.append((s, e))
    with P.Simulator(precision="bf16", sparse24=True, record_rows=True, force_predict=True) as sim:
        sim.load_trace(tr); sim.partition(N, 0); sim.load_model(arch, w); sim.force_latencies(forced)
        sim.simulate()
        agree = n = 0
        errs = []
        for s, e in rows:
            lat, _, _ = sim.get_rows(s, e - s)
            yg = sim.get_outputs(s, e - s)
            errs.append(_rows_err(yg, ref_y[s:e]))
            eq = np.all(lat == forced[s:e], axis=1)
            agree += int(np.sum(eq))
            n += e - s
            for r in np.nonzero(~eq)[0]:          # every disagreement must be a rounding-boundary case (R15)
                assert _legit_flip(yg[r], ref_y[s + r], lat[r], forced[s + r], Y_TOL["bf16"]), (s + r, yg[r], ref_y[s + r])
    errs = np.concatenate(errs)
    print(f"S3 sparse {arch} L={L} N={N}: decisions {agree}/{n}, y err max {errs.max():.2e} median {np.median(errs):.2e}")
    assert errs.max() <= Y_TOL["bf16"] and np.median(errs) <= Y_MEDIAN
    assert agree / n >= 0.99
    # free-running totals (W = 64) vs the oracle on the same sub-traces
    with P.Simulator(precision="bf16", sparse24=True) as sim:
        sim.load_trace(tr); sim.partition(N, 64); sim.load_model(arch, w); sim.simulate()
        cyc = sim.subtrace_cycles()
    js = list(range(N)) if samples is None else samples
    ref_c = sum(int(oracle.simulate(tr, N, 64, arch=arch, weights=w, mode=oracle.BF16, j0=j, nj=1,
                                    want_rows=False)["cycles"][0]) for j in js)
    gpu_c = sum(int(cyc[j]) for j in js)
    assert abs(gpu_c - ref_c) / ref_c <= 0.005, (gpu_c, ref_c)
