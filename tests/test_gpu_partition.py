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
