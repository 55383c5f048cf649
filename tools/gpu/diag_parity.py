"""Diagnose GPU vs oracle latency disagreements (sampled sub-traces)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import oracle, synth
import paper_conf_sc_pandeylfhl22_b200 as P

def run(L, N, W, seed, samples, precision, arch="C3"):
    tr = synth.trace(L, seed)
    w = synth.weights(arch)
    mode = oracle.BF16 if precision == "bf16" else oracle.FP64
    with P.Simulator(precision=precision, record_rows=True) as sim:
        sim.load_trace(tr); sim.partition(N, W); sim.load_model(arch, w); sim.simulate()
        cyc = sim.subtrace_cycles()
        for j in samples:
            t = time.time()
            ref = oracle.simulate(tr, N, W, arch=arch, weights=w, j0=j, nj=1, mode=mode)
            s, e = j * L // N, (j + 1) * L // N
            lat, k, clk = sim.get_rows(s, e - s)
            rl = ref["lat"][s:e]
            eq = np.all(lat == rl, axis=1)
            mism = np.nonzero(~eq)[0]
            info = ""
            if len(mism):
                i0 = mism[0]
                y = ref["y"][s + i0]
                info = f"first mismatch row {i0}: gpu {lat[i0]} oracle {rl[i0]} oracle_y {y} k {ref['k'][s+i0]} vs {k[i0]}"
            print(f"{precision} {arch} L={L} N={N} W={W} j={j}: agree {eq.mean():.5f} ({len(mism)} mism of {e-s}) "
                  f"cycles gpu {cyc[j]} oracle {ref['cycles'][0]} ({time.time()-t:.1f}s) {info}", flush=True)
            if len(mism):
                # CNN-only check at the first mismatch: same input X through both
                q = oracle.Queue(110)
                ws = max(0, s - W)
                for i in range(ws, s + i0 + 1):
                    X, kk = q.build_input(tr, i)
                    if i == s + i0:
                        yg = sim.cnn_forward(X[None])[0]
                        yo = oracle.cnn_forward(arch, w, X, mode=mode)
                        print(f"   same-input CNN at mismatch: gpu {yg} oracle {yo} diff {yg - yo}", flush=True)
                    q.update(i, *(int(v) for v in ref["lat"][i]) if i >= s else
                             tuple(oracle.round_latency(v) for v in oracle.cnn_forward(arch, w, X, mode=mode)))

run(1_000_000, 1024, 1000, synth.TRACE_SEED_BASE + 1, [0, 517, 1023, 640, 700, 967], "bf16")
run(20_000, 8, 64, 77, [0, 3, 7], "bf16")
run(20_000, 8, 64, 77, [0, 3], "fp32")
run(10_000, 1, 0, synth.TRACE_SEED_BASE, [0], "fp32", arch="M2")
