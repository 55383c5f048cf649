"""Host-side logic of bench.py (CPU): the algorithmic FLOP counts behind the
roofline fraction and the roofline arithmetic."""
import bench


def test_flop_counts_from_layer_shapes():
    # conv1: 4 positions x 2 x (2 taps x 50 real features) x 64; conv2: 2 x 2 x 128 x 128;
    # conv3: 2 x 256 x 128 (C3 shapes, R11)
    assert bench.CONV1_FLOP == 51_200
    assert bench.CONV2_FLOP == 65_536
    assert bench.CONV3_FLOP == 65_536
    assert bench.CONV_STACK_FLOP_PER_BLOCK == 182_272
    # full constant folding = 247,808 * P + 1,536 per instruction
    assert bench.CONV_STACK_FLOP_PER_BLOCK + bench.FC1_FLOP_PER_BLOCK == 247_808
    assert bench.step_flops(3, 1) == 247_808 * 3 + 1_536


def _stats(conv_ms, fc_ms, steps, blocks_per_step, n):
    return {"kernel_names": ["gemm_layer0", "gemm_layer1", "gemm_layer2", "gemm_layer3", "gather", "update",
                             "head", "other"],
            "kernel_ms": [conv_ms, 0, 0, fc_ms, 0, 0, 0, 1.0],
            "kernel_launches": [steps, 0, 0, steps, 0, 0, 0, 4],
            "k_hist": [0] * 112, "layer_m": [blocks_per_step, 0, 0, n], "layer_n": [128, 0, 0, 256],
            "layer_k": [0, 0, 0, 512000], "subtraces": n, "simulated": n * steps, "steps": steps,
            "sim_ms": conv_ms + fc_ms + 1.0}


def test_roofline_frac_reproducible():
    steps, bps, n = 1000, 200_000, 65536
    st = _stats(80.0, 30.0, steps, bps, n)
    r = bench.roofline(st, 1, {"arch": "C3", "precision": "bf16"})
    peak = r["peak"]
    avg_s = 80.0 / 1e3 / steps
    want = bps * 182_272 / avg_s / 1e12 / peak
    assert abs(r["frac"] - want) < 1e-3
    assert r["kernel"].startswith("conv_stack")
    step_s = 111.0 / 1e3 / steps
    assert abs(r["step"]["frac"] - (bps * 247_808 + n * 1536) / step_s / 1e12 / peak) < 1e-3


def test_roofline_rb7_counts_all_tensor_kernels():
    """RB7 (config 5): the fused gather + stem, residual-block and fc1 kernels are reported
    together against 10.81 MFLOP per simulated instruction, with no DRAM
    figure borrowed from a C3 capture."""
    steps, n = 100, 4096
    st = {"kernel_names": ["gemm_layer0", "gemm_layer1", "gemm_layer2", "gemm_layer3", "gather", "update",
                           "head", "other"],
          "kernel_ms": [10.0, 20.0, 0, 30.0, 0, 5.0, 1.0, 0.5],
          "kernel_launches": [steps, steps, 0, 3 * steps, 0, steps, steps, 2],
          "k_hist": [0] * 112, "layer_m": [n * 58, n * 58, 0, n], "layer_n": [64, 64, 0, 256],
          "layer_k": [128, 192, 0, 3712], "subtraces": n, "simulated": n * steps, "steps": steps, "sim_ms": 66.5}
    r = bench.roofline(st, 1, {"arch": "RB7", "precision": "bf16"})
    flop = n * steps * (2 * 56 * 100 * 64 + 6 * 2 * 56 * 192 * 64 + 2 * 3584 * 256)
    assert flop == n * steps * 10_809_344
    want = flop / 60e-3 / 1e12 / r["peak"]
    assert abs(r["frac"] - want) < 1e-3
    assert "resblock" in r["kernel"] and r["traffic"] is None
