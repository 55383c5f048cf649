"""2:4 magnitude pruning of the synthetic weights (R22).

Pruning is model preparation: both the oracle and the GPU load the pruned weights
unchanged (the oracle's dense CNN on them is exact).  Pinned here against its definition:
in every group of 4 consecutive inputs along each tensor-core layer's reduction dimension
in the DEVICE order (conv: input channels of one tap; linear: flattened inputs) at most 2
weights are nonzero, they are the 2 largest magnitudes of the dense weights (ties: lower
index), and the fc2 head is untouched."""
import numpy as np
import pytest

import synth


def _layers(w, arch):
    out, off = [], 0
    for ws, bs in synth.layer_shapes(arch):
        n = int(np.prod(ws))
        out.append((w[off:off + n].reshape(ws), w[off + n:off + n + int(np.prod(bs))]))
        off += n + int(np.prod(bs))
    return out


def _groups(wl):
    """[..., 4] groups along the device reduction order."""
    if wl.ndim == 3:                                   # conv [Cout][Cin][k] -> [Cout][k][Cin]
        v = np.moveaxis(wl, 2, 1)
    else:
        v = wl[:, None, :]
    pad = (-v.shape[2]) % 4
    if pad:
        v = np.concatenate([v, np.zeros(v.shape[:2] + (pad,))], axis=2)
    return v.reshape(v.shape[0], v.shape[1], -1, 4)


@pytest.mark.parametrize("arch", ["C3", "M2"])
def test_pruned_layers_are_2_of_4_and_keep_the_largest(arch):
    dense = _layers(synth.weights(arch).astype(np.float64), arch)
    # the pruned file uses its own head calibration; compare the tensor-core layers only
    sparse = _layers(synth.weights(arch, sparse24=True).astype(np.float64), arch)
    for li, ((wd, bd), (wsp, bsp)) in enumerate(zip(dense[:-1], sparse[:-1])):
        gd, gs = _groups(wd), _groups(wsp)
        nz = np.count_nonzero(gs, axis=3)
        assert nz.max() <= 2
        # kept weights equal the dense ones where kept
        mask = gs != 0
        assert np.array_equal(gs[mask], gd[mask].astype(np.float32).astype(np.float64))
        # and they are the 2 largest magnitudes of each group (brute force per group)
        ad = np.abs(gd).reshape(-1, 4)
        ks = mask.reshape(-1, 4)
        for row in range(0, ad.shape[0], max(1, ad.shape[0] // 2000)):
            want = sorted(sorted(range(4), key=lambda t: (-ad[row, t], t))[:2])
            got = [t for t in range(4) if ks[row, t]]
            assert set(got) <= set(want), (li, row, got, want)
        assert np.array_equal(bd, bsp)                 # biases are not pruned
    assert sparse[-1][0].shape == (3, 256) and np.count_nonzero(sparse[-1][0]) > 256 * 3 // 2   # head dense


def test_prune24_on_a_hand_example():
    w = np.array([[[3.0, 0.0], [-5.0, 1.0], [1.0, -2.0], [0.5, 0.5], [7.0, 1.0]]])   # [1][5][2]
    p = synth.prune24(w, "conv")
    # tap 0: channels 0..3 = (3, -5, 1, 0.5) -> keep -5, 3; channel 4 alone (group of 1) kept
    assert p[0, :, 0].tolist() == [3.0, -5.0, 0.0, 0.0, 7.0]
    # tap 1: (0, 1, -2, 0.5) -> keep -2, 1
    assert p[0, :, 1].tolist() == [0.0, 1.0, -2.0, 0.0, 1.0]
    lin = synth.prune24(np.array([[1.0, 1.0, 1.0, 2.0]]), "linear")   # tie: lower index kept
    assert lin.tolist() == [[1.0, 0.0, 0.0, 2.0]]
