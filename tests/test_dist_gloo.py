"""World-size-2 CPU test (gloo) of the multi-GPU host logic: each rank takes its
contiguous sub-trace block from psim_partition_range, sees only its own trace
rows (warm-up halo included), simulates them, and the int64 totals are summed
with the same all-reduce helper bench.py uses.  The sum must equal the
single-process total bit-exactly (sub-traces are independent).
The per-rank simulation here is the oracle (no GPU on this box); on the GPU
the same host logic drives libpsim (test_gpu_parity rank-slice test)."""
import os
import socket

import numpy as np
import torch.multiprocessing as mp

import oracle
import paper_conf_sc_pandeylfhl22_b200 as P
import synth

L, N, W = 6000, 37, 45


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    rr = P.partition_range(L, N, W, rank, world)
    rows = synth.trace(rr.row_hi - rr.row_lo, 5, r0=rr.row_lo)        # only this rank's rows
    lat = synth.teacher_latencies(L, 8, big=0.01)
    out = oracle.simulate(rows, N, W, forced_lat=lat, j0=rr.j0, nj=rr.j1 - rr.j0, L=L, row_offset=rr.row_lo,
                          want_rows=False)
    total = P.all_reduce_total(out["total"])
    q.put((rank, rr.j0, rr.j1, out["total"], total))
    dist.destroy_process_group()


def test_two_rank_gloo_total_matches_single_process():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    tr = synth.trace(L, 5)
    lat = synth.teacher_latencies(L, 8, big=0.01)
    ref = oracle.simulate(tr, N, W, forced_lat=lat, want_rows=False)
    assert res[0][1] == 0 and res[0][2] == res[1][1] and res[1][2] == N     # contiguous blocks cover N
    assert res[0][3] + res[1][3] == ref["total"]
    assert res[0][4] == res[1][4] == ref["total"]
