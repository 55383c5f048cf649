"""bench.py -- parallel sub-trace ML simulation throughput on B200 (MIPS).

    python bench.py [--gpus N --steps K --warmup W] [--impl psim|reference] [--config c3|c2|c1]

A step is one pass of the whole hot path -- psim_simulate: every lockstep step
of gather -> CNN GEMMs -> head -> round/update over all sub-traces, then the
cycle reduction (+ NCCL all-reduce for N > 1) -- over one synthetic trace.
Default workload: BASELINE.json configs[2] (the metric's config): a
100M-instruction SPEC-like synthetic trace, 65536 sub-traces, W = 110
(= Context_length), C3 CNN, bf16 operands; it fits one GPU.

value  = instructions simulated by all ranks (warm-up excluded) / max-over-ranks
         device time of K steps, trace resident in HBM before the timed region.
e2e    = the same through psim_load_trace with a PINNED HOST trace: the H2D copy
         of each rank's rows and the D2H of the total are inside every step.
roofline / cpu_baseline / clocks: see DESIGN.md "measurement".

Under torchrun (N > 1) each rank owns the contiguous sub-trace block
[g N/G, (g+1) N/G) and generates only its own trace rows (counter-based
generator), so nothing but the final int64 cycle count crosses NVLink.
"""
from __future__ import annotations

import argparse
import json
import os
import signal
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    "c1": dict(L=10_000, N=1, W=0, arch="M2", precision="fp32", seed_off=0,
               desc="config1: 10k-instruction synthetic trace, 1 sub-trace, queue 111, M2 CNN, fp32"),
    "c2": dict(L=1_000_000, N=1024, W=1000, arch="C3", precision="bf16", seed_off=1,
               desc="config2: 1M-instruction synthetic SPEC-like trace, 1024 sub-traces, W=1000, C3 CNN, bf16"),
    "c3": dict(L=100_000_000, N=65536, W=110, arch="C3", precision="bf16", seed_off=2,
               desc="config3: 100M-instruction synthetic SPEC-like trace, 65536 sub-traces, W=110, C3 CNN, bf16"),
    # BASELINE.json configs[4]: 1B instructions, deeper residual CNN, 8 GPUs, streamed loading.
    # [proposal, SURVEY §8d] N = 262144, W = 1000 -> 3815 instructions per sub-trace.
    "c5": dict(L=1_000_000_000, N=262144, W=1000, arch="RB7", precision="bf16", seed_off=4,
               desc="config5: 1B-instruction synthetic SPEC-like trace, 262144 sub-traces, W=1000, RB7 CNN, bf16"),
    # one GPU's share of config 5 at 8 GPUs (32768 sub-traces of 3815 instructions, W=1000)
    "c5s": dict(L=125_000_000, N=32768, W=1000, arch="RB7", precision="bf16", seed_off=4,
                desc="config5 per-GPU slice: 125M-instruction trace, 32768 sub-traces, W=1000, RB7 CNN, bf16"),
    # profiling stand-in: config 3's batch shape (65536 sub-traces, W=110) on a 4.2M-row
    # prefix -> 174 lockstep steps with the same per-step kernel shapes (ncu runs only)
    "c3p": dict(L=65536 * 64, N=65536, W=110, arch="C3", precision="bf16", seed_off=2,
                desc="profiling: config3 batch shape on a 4.2M-row prefix (65536 sub-traces, W=110), C3, bf16"),
}
METRIC = "simulated instr/sec (MIPS, 8×B200 device-timed) + cycle error vs CPU oracle"
REASONS = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# --------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi sampling DURING the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = "index,clocks.sm,clocks.max.sm,power.draw," + ",".join(f"clocks_event_reasons.{r}" for r in REASONS)
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={index}", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                       "-lms", "100"], stdout=self.f, stderr=subprocess.DEVNULL, start_new_session=True)
        except FileNotFoundError:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        os.killpg(self.p.pid, signal.SIGTERM)
        self.p.wait()
        self.f.flush()
        rows = [l.split(",") for l in open(self.f.name).read().strip().splitlines() if l.strip()]
        os.unlink(self.f.name)
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if r[1].strip().replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].strip().replace(".", "").isdigit()]
        reasons = sorted({REASONS[i] for r in rows for i in range(len(REASONS))
                          if len(r) > 4 + i and "Active" in r[4 + i] and "Not" not in r[4 + i]})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


# --------------------------------------------------------------------------- roofline
# Algorithmic FLOP of the fused C3 path (SURVEY.md §8(d) "full constant-folding" count,
# DESIGN.md §5), per block (sub-trace b, conv3 position p < P_b) and per sub-trace:
CONV1_FLOP = 4 * 2 * 100 * 64      # 4 conv1 positions per block; K = 2 taps x 50 real features
CONV2_FLOP = 2 * 2 * 128 * 128     # 2 conv2 positions; K = 2 taps x 64 channels
CONV3_FLOP = 2 * 256 * 128         # 1 conv3 position; K = 2 taps x 128 channels
CONV_STACK_FLOP_PER_BLOCK = CONV1_FLOP + CONV2_FLOP + CONV3_FLOP   # 182,272
FC1_FLOP_PER_BLOCK = 2 * 128 * 256  # fc1 over the P_b computed positions (x 128 channels)
FC2_FLOP_PER_SUBTRACE = 2 * 256 * 3


def step_flops(blocks_per_step, n_active):
    """Algorithmic FLOP of one lockstep step: 247,808 per block + 1,536 per sub-trace."""
    return blocks_per_step * (CONV_STACK_FLOP_PER_BLOCK + FC1_FLOP_PER_BLOCK) + n_active * FC2_FLOP_PER_SUBTRACE


def roofline(stats, k_steps, cfg):
    """Dominant kernel class by device time; algorithmic work per launch / average
    launch duration (CUDA events on the launch stream, PSIM_PROFILE)."""
    names, ms, launches = stats["kernel_names"], stats["kernel_ms"], stats["kernel_launches"]
    total_ms = sum(ms)
    dom = int(np.argmax(ms))
    pk, src = peaks()
    out = {"kernel": names[dom], "share": round(ms[dom] / total_ms, 4) if total_ms else None}
    avg_s = ms[dom] / 1e3 / max(launches[dom], 1)
    hist = np.array(stats["k_hist"], np.float64)
    kmean = float((hist * np.arange(112)).sum() / max(hist.sum(), 1))
    fused = stats["layer_k"][0] == 0 and stats["layer_m"][0] > 0   # fused path: conv_stack + fc1_head
    sustained = pk["bf16_tflops_sustained"]
    if cfg["arch"] == "RB7" and names[dom].startswith("gemm_layer"):
        # the RB7 tensor-core kernels, reported together (5 launches per step: gather + stem
        # fused, 3 residual blocks, fc1): stem 2*56*100*64 + six k3 convs 6 * 2*56*192*64 + fc1
        # 2*3584*256 per simulated instruction
        g = [i for i in range(len(names)) if names[i].startswith("gemm_layer")]
        g_ms = sum(ms[i] for i in g)
        flops = float(stats["simulated"]) * k_steps * (716800 + 6 * 1376256 + 1835008)
        achieved = flops / (g_ms / 1e3) / 1e12
        out.update(kernel="rb7_stem_kernel + resblock_kernel x3 + gemm_tc_kernel (fc1): all RB7 layers", share=round(g_ms / total_ms, 4), bound="tensor",
                   achieved=round(achieved, 2), peak=sustained, unit="TFLOP/s", frac=round(achieved / sustained, 4),
                   flops_per_step=flops / k_steps, peak_source=src + " bf16_tflops_sustained")
        avg_s = g_ms / 1e3 / max(sum(launches[i] for i in g), 1)
    elif names[dom].startswith("gemm_layer"):
        li = int(names[dom][-1])
        M, N, K = stats["layer_m"][li], stats["layer_n"][li], stats["layer_k"][li]
        if fused and li == 0:     # conv_stack: M = mean blocks per step (= per launch)
            flops = float(M) * CONV_STACK_FLOP_PER_BLOCK
        elif fused and li == 3:   # fc1_head: fc1 over the P_b computed positions of each sub-trace + fc2
            flops = float(stats["layer_m"][0]) * FC1_FLOP_PER_BLOCK + float(M) * FC2_FLOP_PER_SUBTRACE
        else:
            k_alg = 100 if li == 0 else K      # conv1: 2 rows x 50 real features (features padded to 64)
            flops = 2.0 * M * N * k_alg
        achieved = flops / avg_s / 1e12
        peak = sustained if cfg["precision"] == "bf16" else 74.0
        out.update(bound="tensor", achieved=round(achieved, 2), peak=peak, unit="TFLOP/s",
                   frac=round(achieved / peak, 4), flops_per_launch=flops,
                   flops_per_unit=(CONV_STACK_FLOP_PER_BLOCK if (fused and li == 0) else None),
                   unit_of_work=("block (sub-trace, conv3 position p < P_b)" if (fused and li == 0) else None),
                   peak_source=(src + " bf16_tflops_sustained") if cfg["precision"] == "bf16" else "derived fp32 SIMT")
    else:
        n = stats["subtraces"]
        if names[dom] == "gather":   # X write (bf16 112x64) + trace rows (k+1)x48 + queue (k x 12 B)
            byts = n * (112 * 64 * 2 + (kmean + 1) * 48 + kmean * 12)
        else:                        # update: queue read+write (2 x k x 12 B) + state + y
            byts = n * (2 * (kmean + 1) * 12 + 64)
        achieved = byts / avg_s / 1e9
        out.update(bound="hbm", achieved=round(achieved, 1), peak=pk["hbm_gbs"], unit="GB/s",
                   frac=round(achieved / pk["hbm_gbs"], 4), bytes_per_launch=byts, peak_source=src + " hbm")
    # DRAM bytes of an ncu capture of the dominant kernel (profiles/ncu_traffic.json: C3 captures only)
    out["traffic"] = None if cfg["arch"] == "RB7" else ncu_traffic(names[dom])
    out["avg_launch_us"] = round(avg_s * 1e6, 2)
    if fused:
        out["kernel"] = {"gemm_layer0": "conv_stack_kernel (gather+conv1+conv2+conv3, fused)",
                         "gemm_layer3": "fc1_head_kernel (fc1+head+update, fused)"}.get(names[dom], names[dom])
        # whole lockstep step: all algorithmic FLOP of the step / mean step time (sim_ms / steps)
        bps = float(stats["layer_m"][0])
        n_act = float(stats["simulated"]) / max(stats["steps"], 1)
        fl = step_flops(bps, n_act)
        step_s = stats["sim_ms"] / 1e3 / max(stats["steps"], 1)
        out["step"] = {"flops": fl, "ms": round(step_s * 1e3, 5), "achieved": round(fl / step_s / 1e12, 2),
                       "frac": round(fl / step_s / 1e12 / sustained, 4), "blocks": round(bps, 1),
                       "note": "algorithmic FLOP of a mean lockstep step (247,808 per block + 1,536 per active "
                               "sub-trace) / (simulate device time / steps), whole simulate incl. reduction"}
    out["kernels"] = {names[i]: {"ms": round(ms[i] / k_steps, 3), "launches": launches[i] // k_steps,
                                 "share": round(ms[i] / total_ms, 4) if total_ms else None}
                      for i in range(len(names)) if launches[i]}
    out["k_mean"] = round(kmean, 2)
    return out


def ncu_traffic(kernel_class):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        d = json.load(open(p))
        v = d.get(kernel_class)
        return v.get("dram_bytes_per_launch") if isinstance(v, dict) else v
    return None


# --------------------------------------------------------------------------- CPU oracle
def oracle_sample(cfg, tr_rows, row_lo, budget_s, L, N, W, j_list=None, seed=7, sparse=False):
    """Run the oracle (as it stands, single thread) on whole sub-traces of the same
    workload until ~budget_s of CPU time; returns (instructions, seconds, cycles)."""
    import oracle
    import synth
    w = synth.weights(cfg["arch"], sparse24=sparse)
    mode = oracle.BF16 if cfg["precision"] == "bf16" else oracle.FP64
    rng = np.random.default_rng(seed)
    done, t_used, per = 0, 0.0, {}
    js = list(j_list) if j_list is not None else []
    while True:
        if j_list is None:
            j = int(rng.integers(0, N))
        else:
            if not js:
                break
            j = js.pop(0)
        s, e = j * L // N, (j + 1) * L // N
        ws = max(0, s - W)
        if tr_rows is not None and ws >= row_lo and e - row_lo <= tr_rows.shape[0]:
            sl = tr_rows[ws - row_lo:e - row_lo]
        else:
            sl = synth.trace(e - ws, synth.TRACE_SEED_BASE + cfg["seed_off"], r0=ws)
        t0 = time.perf_counter()
        r = oracle.simulate(sl, N, W, arch=cfg["arch"], weights=w, mode=mode, j0=j, nj=1, L=L, row_offset=ws,
                            want_rows=False)
        t_used += time.perf_counter() - t0
        done += e - s
        per[j] = int(r["cycles"][0])
        if j_list is None and t_used >= budget_s:
            break
    return done, t_used, per


def _oracle_worker(args):
    """One all-core oracle process: whole random sub-traces for ~budget_s of its own CPU."""
    cfg_name, budget_s, seed, sparse = args
    cfg = CONFIGS[cfg_name]
    os.environ.setdefault("OMP_NUM_THREADS", "1")
    n_i, t, per = oracle_sample(cfg, None, 0, budget_s, cfg["L"], cfg["N"], cfg["W"], seed=seed, sparse=sparse)
    return n_i, t, len(per)


def host_info():
    info = {"nproc": len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        keep = ("Model name", "Socket(s)", "Core(s) per socket", "Thread(s) per core", "CPU(s)", "CPU max MHz")
        for ln in out.splitlines():
            k, _, v = ln.partition(":")
            if k.strip() in keep:
                info["lscpu " + k.strip()] = v.strip()
    except Exception as ex:  # noqa: BLE001 - informational only
        info["lscpu"] = f"unavailable: {ex}"
    return info


def oracle_all_cores(cfg_name, budget_s, sparse=False):
    """The oracle as it stands on every host core: P = nproc independent processes, each
    simulating whole random sub-traces of the same workload for ~budget_s.  Returns
    (instructions, wall seconds, P, sub-traces)."""
    import multiprocessing as mp
    P = host_info()["nproc"]
    ctx = mp.get_context("spawn")
    t0 = time.perf_counter()
    with ctx.Pool(P) as pool:
        res = pool.map(_oracle_worker, [(cfg_name, budget_s, 1000 + i, sparse) for i in range(P)])
    wall = time.perf_counter() - t0
    # per-process throughput is measured on its own clock; aggregate = sum of per-process rates
    rate = sum(n / t for n, t, _ in res if t > 0)
    return sum(n for n, _, _ in res), wall, P, sum(c for _, _, c in res), rate


# --------------------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="psim", choices=["psim", "reference"])
    ap.add_argument("--config", default="c3", choices=sorted(CONFIGS))
    ap.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of single-thread oracle work for cpu_baseline")
    ap.add_argument("--cpu-budget-all", type=float, default=12.0,
                    help="seconds per process of the all-core oracle run (P = nproc processes)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg (profiling runs)")
    ap.add_argument("--emulate-rank", default=None, metavar="R/G",
                    help="diagnostics: run rank R's share of a G-GPU job on this one GPU (no NCCL), "
                         "to estimate per-GPU throughput at G GPUs; value = that rank's instructions/s")
    ap.add_argument("--sparse", action="store_true",
                    help="2:4 structured sparsity (PAPER.md:157): 2:4-pruned weights on the sparse tcgen05.mma.sp "
                         "layer-wise path (PSIM_SPARSE24)")
    ap.add_argument("--layerwise", action="store_true",
                    help="run the layer-by-layer tcgen05 GEMM path instead of the fused kernels (A/B)")
    ap.add_argument("--correction", type=int, default=0,
                    help="post-error correction limit (PAPER.md:203-219; the paper uses 100); 0 = off")
    args = ap.parse_args()
    cfg = CONFIGS[args.config]
    L, N, W = cfg["L"], cfg["N"], cfg["W"]

    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # started without torchrun: launch one rank per GPU ourselves (same arguments)
        import socket
        with socket.socket() as so:
            so.bind(("127.0.0.1", 0))
            port = so.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
        log("[bench] launching", " ".join(cmd))
        sys.exit(subprocess.call(cmd))
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus and args.impl != "reference":
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}; launch one rank per GPU")
    emu = None
    if args.emulate_rank:
        emu = tuple(int(x) for x in args.emulate_rank.split("/"))   # (R, G): partition as rank R of G
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    config = {"workload": cfg["desc"], "instructions": L, "subtraces": N, "warmup_W": W, "cnn": cfg["arch"],
              "queue_rows": 111, "precision": cfg["precision"],
              "l2": "inputs larger than L2 (trace %.1f GB resident in HBM)" % (L * 48 / 1e9),
              "post_error_correction": args.correction}
    if args.sparse:
        config["sparsity"] = "2:4 magnitude-pruned tensor-core layers, tcgen05.mma.sp layer-wise path (R22)"
    if args.layerwise:
        config["path"] = "layer-wise tcgen05 GEMMs"

    if args.impl == "reference":
        # the oracle as it stands, on rank 0 only, on the host cores
        if rank != 0:
            return
        # every step: P = nproc oracle processes (a persistent pool) each simulate whole random
        # sub-traces of the workload for ~per_step seconds; step time = wall clock of the step
        import multiprocessing as mp
        hi = host_info()
        P = hi["nproc"]
        per_step = float(os.environ.get("PSIM_REF_STEP_S", "3.0"))
        times, insts, subs = [], 0, 0
        with mp.get_context("spawn").Pool(P) as pool:
            for it in range(args.warmup + args.steps):
                t0 = time.perf_counter()
                res = pool.map(_oracle_worker, [(args.config, per_step, 100000 * it + i, args.sparse) for i in range(P)])
                dt = time.perf_counter() - t0
                if it >= args.warmup:
                    times.append(dt); insts += sum(r[0] for r in res); subs += sum(r[2] for r in res)
        tot = sum(times)
        val = insts / tot / 1e6
        line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "MIPS", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic", "config": config,
                "cpu_baseline": {"value": val, "unit": "MIPS", "cores": P, "kind": "oracle",
                                 "sample": f"per step: {P} processes x ~{per_step:.0f} s of whole random sub-traces "
                                           f"of {args.config} ({insts} counted instructions, {subs} sub-traces over "
                                           f"{args.steps} timed steps), plain-C oracle "
                                           + ("bf16-operand" if cfg["precision"] == "bf16" else "fp64") + " mode",
                                 "host": hi},
                "e2e": {"value": val, "unit": "MIPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_sc_pandeylfhl22_b200 as P
    import synth

    torch.cuda.set_device(local_rank)
    if world > 1:
        # NCCL's communicator-init lines (rank / nranks / transport) on stderr, so a multi-GPU
        # run shows its ranks; stdout keeps the one JSON line
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    nccl_id = None
    if world > 1:
        obj = [P.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        nccl_id = obj[0]

    rr = P.partition_range(L, N, W, *(emu if emu else (rank, world)))
    rows = rr.row_hi - rr.row_lo
    t0 = time.time()
    host = torch.empty((rows, 48), dtype=torch.uint8, pin_memory=True)
    synth.trace_into(host.numpy(), synth.TRACE_SEED_BASE + cfg["seed_off"], rr.row_lo)
    dev = host.cuda()
    w = synth.weights(cfg["arch"], sparse24=args.sparse)
    log(f"[rank {rank}] trace rows [{rr.row_lo},{rr.row_hi}) generated in {time.time() - t0:.1f}s")

    stream = torch.cuda.Stream()

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    sim = P.Simulator(device=local_rank, precision=cfg["precision"], rank=emu[0] if emu else rank,
                      world_size=emu[1] if emu else world, nccl_id=nccl_id,
                      stream=stream.cuda_stream, profile=os.environ.get("PSIM_NOPROF") is None, chunk_steps=int(os.environ.get("PSIM_CHUNK", "0")),
                      correction_limit=args.correction, sparse24=args.sparse, layerwise=args.layerwise)
    sim.load_model(cfg["arch"], w)

    def timed(trace_tensor, k_steps, warm):
        sim.load_trace(trace_tensor, n_instr=L, first_row=rr.row_lo)
        sim.partition(N, W)
        for _ in range(warm):
            sim.simulate()
        barrier()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        clk = ClockSampler(local_rank)
        ev0.record(stream)
        tot = None
        kms = None
        for _ in range(k_steps):
            sim.simulate()
            tot = sim.total_cycles()            # D2H of the step's result
            st = sim.stats()
            kms = st if kms is None else {**st, "kernel_ms": [a + b for a, b in zip(kms["kernel_ms"], st["kernel_ms"])],
                                          "kernel_launches": [a + b for a, b in zip(kms["kernel_launches"], st["kernel_launches"])]}
        ev1.record(stream)
        barrier()
        clocks = clk.stop()
        ms = ev0.elapsed_time(ev1)
        return max_over_ranks(ms), tot, kms, clocks

    ms, total, stats, clocks = timed(dev, args.steps, args.warmup)
    value = L * args.steps / (ms / 1e3) / 1e6
    if emu:   # this rank's counted instructions only
        value = stats["counted"] * args.steps / (ms / 1e3) / 1e6
        config["emulated_rank"] = f"{emu[0]}/{emu[1]} (one GPU's share of a {emu[1]}-GPU job, no NCCL)"
    e2e = None
    if not args.no_e2e:
        ms_e, total_e, st_e, _ = timed(host, args.steps, 1)
        assert total_e == total, (total_e, total)
        ranges = [P.partition_range(L, N, W, g, world) for g in range(world)]
        e2e = {"value": L * args.steps / (ms_e / 1e3) / 1e6, "unit": "MIPS",
               "h2d_bytes_per_step": int(sum((x.row_hi - x.row_lo) * 48 for x in ranges)),
               "d2h_bytes_per_step": 8 * world}

    line = {"metric": METRIC, "value": value, "unit": "MIPS", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": cfg["precision"], "data": "synthetic", "config": config,
            "total_cycles": total, "e2e": e2e, "gpu_launches": int(sum(stats["kernel_launches"])),
            "clocks": clocks}
    if world > 1:   # the final ncclAllReduce of the cycle total: ranks of the library's communicator
        line["comm"] = {"backend": "nccl", "ranks": int(stats.get("comm_ranks", 0)), "world_size": world}
    if rank == 0:
        line["roofline"] = roofline(stats, args.steps, cfg) if sum(stats["kernel_ms"]) > 0 else None
        line["stats"] = {k: stats[k] for k in ("steps", "simulated", "counted", "stalls", "subtraces", "corrected",
                                               "corr_steps")}
        line["warmup_overhead"] = round(stats["simulated"] / stats["counted"] - 1, 4)
    if rank == 0 and world == 1 and not args.no_cpu:
        # cpu_baseline: the oracle as it stands on a bounded sample of the same workload,
        # plus the sampled sub-traces' cycles vs the GPU (parity sample)
        n_i, t, per = oracle_sample(cfg, host.numpy(), rr.row_lo, args.cpu_budget, L, N, W, sparse=args.sparse)
        gcyc = sim.corrections()[1] if args.correction else sim.subtrace_cycles()   # first-pass cycles
        errs = [abs(int(gcyc[j]) - c) / max(c, 1) for j, c in per.items()]
        n_all, wall_all, P_all, sub_all, rate_all = oracle_all_cores(args.config, args.cpu_budget_all, args.sparse)
        line["cpu_baseline"] = {"value": rate_all / 1e6, "unit": "MIPS", "cores": P_all, "kind": "oracle",
                                "sample": f"all host cores: {P_all} oracle processes x ~{args.cpu_budget_all:.0f} s, "
                                          f"{sub_all} whole random sub-traces ({n_all} counted instructions, W={W} "
                                          f"warm-up each) of {args.config}; value = sum of per-process rates "
                                          f"(wall {wall_all:.1f} s incl. start-up)",
                                "host": host_info(),
                                "single_thread": {"value": n_i / t / 1e6, "unit": "MIPS", "cores": 1,
                                                  "sample": f"{len(per)} whole sub-traces ({n_i} counted "
                                                            f"instructions) of {args.config}, "
                                                            f"{t:.1f} s"},
                                "mode": "plain-C oracle, " + ("bf16-operand" if cfg["precision"] == "bf16" else "fp64")
                                        + " mode, dense CNN"}
        line["parity_sample"] = {"subtraces": sorted(per), "max_rel_cycle_err": max(errs) if errs else None}
    sim.close()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
