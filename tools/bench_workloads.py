#!/usr/bin/env python
"""Secondary benchmarks (configs 3-5 of BASELINE.json) -- one JSON line per run.

    python tools/bench_workloads.py --workload pagerank|sssp|micro [--scale 24] [--steps K]
           [--warmup W] [--chunk BYTES] [--mech fused] [--ranks G] [--no-cpu]

pagerank: step = 20 PageRank iterations on RMAT-scale (edge factor 16), value = iters/s.
sssp:     step = Bellman-Ford to convergence (rounds as the oracle), value = rounds/s.
micro:    step = one phase of the transfer microbenchmark (R bytes, all-gather shape) over
          --ranks loopback ranks on this GPU; value = replicated bytes/s (HBM-to-HBM here:
          with one GPU there is no NVLink, so this measures the protocol, not the link).
Roofline: the phase kernel's algorithmic bytes per launch / CUDA-event time (DESIGN.md Sec.
"Roofline accounting").  cpu_baseline: the oracle on a bounded sample.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # loopback ranks: see loopback.py
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402


def peak_hbm():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        return 6650.0


def ev():
    return torch.cuda.Event(enable_timing=True)


def pagerank(args, src, dst, V):
    def body(r, G):
        rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[args.mech])
        s = torch.cuda.Stream()
        P = wl.PageRank(V, src, dst, args.chunk, stream=s)
        I = 20

        def step():
            for k in range(I):
                P.step(s, barrier=(k == I - 1))
        for _ in range(args.warmup):
            step()
        torch.cuda.synchronize()
        e0, e1 = ev(), ev()
        e0.record(s)
        for _ in range(args.steps):
            step()
        e1.record(s)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        ks = []
        for _ in range(10):
            a, b = ev(), ev()
            i = P.k & 1
            a.record(s)
            _lib.check(rt.lib().proact_pagerank_phase(P.gid, P.rid[i], P.rid[i ^ 1], P.d, wl._s(s)), "pr")
            b.record(s)
            rt.phase_sync(s)
            P.k += 1
            ks.append((a, b))
        torch.cuda.synchronize()
        kms = statistics.median(a.elapsed_time(b) for a, b in ks)
        out = {"ms": ms, "kms": kms, "e_own": P.e_own, "nv": P.v1 - P.v0, "iters": args.steps * I,
               "nhot": P.nhot, "e_hot": P.e_hot}
        if G == 1:   # tracking overhead (Fig. 8 methodology): tallies + agent, pushes elided, vs LOCAL
            def phase_ms(mech, n=10):
                rt.set_config(mech=mech)
                torch.cuda.synchronize()
                a, b = ev(), ev()
                a.record(s)
                for _ in range(n):
                    P.step(s)
                b.record(s)
                torch.cuda.synchronize()
                return a.elapsed_time(b) / n
            w0 = rt.get_config()["agent_warps"]
            phase_ms(_lib.MECH_ELIDE, 2)
            out["overhead"] = {"local_ms": phase_ms(_lib.MECH_LOCAL), "elide_ms": phase_ms(_lib.MECH_ELIDE),
                               "agent_warps": w0}
            rt.set_config(agent_warps=4)   # PageRank pushes 4 B/vertex: a few agent CTAs suffice
            phase_ms(_lib.MECH_ELIDE, 2)
            out["overhead"]["elide4_ms"] = phase_ms(_lib.MECH_ELIDE)
            rt.set_config(agent_warps=w0, mech={v: k for k, v in _lib.MECH_NAMES.items()}[args.mech])
        P.free()
        return out
    res = run_ranks(args.ranks, body)
    ms = max(r["ms"] for r in res)
    kms = max(r["kms"] for r in res)
    alg = max(8.0 * r["e_own"] + 16.0 * r["nv"] for r in res)
    line = {"workload": f"pagerank_rmat{args.scale}_ef16_20it (BASELINE.json config 3)",
            "value": res[0]["iters"] / (ms / 1000.0), "unit": "iters/s", "ranks": args.ranks,
            "mech": args.mech, "chunk_bytes": args.chunk, "edges": int(src.size),
            "roofline": {"bound": "hbm", "kernel": "pagerank_hot_kernel" if res[0]["nhot"] else "pagerank_kernel",
                         "kernel_ms": kms, "hot_sources": res[0]["nhot"], "hot_edge_frac": res[0]["e_hot"] / max(1, res[0]["e_own"]),
                         "alg_bytes_per_launch": alg, "achieved": alg / kms / 1e6, "peak": peak_hbm(),
                         "unit": "GB/s", "frac": alg / kms / 1e6 / peak_hbm(),
                         "note": "8 B/edge (index + gathered contrib) + 16 B/vertex; gathers hit L2"}}
    # the bound that actually applies: every random 4-byte gather from global
    # memory is one L1TEX wavefront / L1->L2 request, one per clock per SM -> t >= gathers /
    # (SMs x SM clock); in-edges of hot sources read shared memory instead
    prop = torch.cuda.get_device_properties(0)
    e_max = max(r["e_own"] - r["e_hot"] for r in res)
    rate = prop.multi_processor_count * 1965e6          # gathers/s at the max SM clock
    t_l1 = e_max / rate * 1e3
    line["roofline_l1_gather"] = {"bound": "l1tex_wavefronts", "gathers_per_launch": e_max,
                                  "peak_gathers_per_s": rate, "t_min_ms": t_l1, "frac": t_l1 / kms,
                                  "note": "global gathers (in-edges of non-hot sources); 1 wavefront/clk/SM x SMs x 1965 MHz"}
    # the same bound MEASURED: tools/probes/gather_peak.cu (an index stream + random 4-byte gathers
    # from a 64 MiB L2-resident vector and nothing else, the best CTA shape), on a B200 of this pool
    try:
        gp = max(json.loads(l)["gathers_per_s"] for l in open(os.path.join(ROOT, "profiles", "r02p_gather_peak.jsonl"))
                 if l.startswith("{"))
        line["roofline_gather_measured"] = {"bound": "random 4-byte gathers (measured)", "peak_gathers_per_s": gp,
                                            "t_min_ms": e_max / gp * 1e3, "frac": e_max / gp * 1e3 / kms,
                                            "source": "profiles/r02p_gather_peak.jsonl (tools/probes/gather_peak.cu)"}
    except (OSError, ValueError):
        pass
    if "overhead" in res[0]:
        o = res[0]["overhead"]
        line["overhead"] = {"local_ms_per_phase": o["local_ms"], "elide_ms_per_phase": o["elide_ms"],
                            "tracking_overhead_frac": o["elide_ms"] / o["local_ms"] - 1.0,
                            "agent_warps": o["agent_warps"],
                            "tracking_overhead_frac_4_agent_warps": o["elide4_ms"] / o["local_ms"] - 1.0,
                            "note": "G=1: ELIDE keeps tallies + agent with remote stores skipped (Fig. 8 methodology)"}
    if not args.no_cpu:
        import oracle
        tm = {}
        oracle.pagerank(V, src, dst, 20, timing=tm)   # the GPU step's 20 iterations
        line["cpu_baseline"] = {"value": 20 / tm["iter_seconds"], "unit": "iters/s",
                                "cores": oracle.get_threads(), "kind": "oracle",
                                "sample": "oracle.pagerank, 20 iterations of the full graph on all "
                                          "host cores (OpenMP); the CSC build is excluded (input preparation)"}
    return line


def sssp(args, src, dst, V):
    w = synth.weights(src.size)
    s0 = int(np.bincount(src, minlength=V).argmax())

    def body(r, G):
        rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[args.mech])
        st = torch.cuda.Stream()
        rounds = None
        times = []
        S = wl.SSSP(V, src, dst, w, s0, args.chunk, stream=st)
        for k in range(args.warmup + args.steps):
            S.reset()
            rt.host_barrier()
            t0 = time.perf_counter()
            rounds = S.run(stream=st)
            times.append(time.perf_counter() - t0)
        # one more run, round by round: the phase kernel's CUDA-event time and its algorithmic
        # bytes (4 B per in-edge scanned + 8 B per in-edge of a source whose
        # chunk changed in the previous round + 12 B per vertex), the changed chunks read back
        # from the distance vectors between rounds (outside the timed kernel)
        S.reset()
        rt.host_barrier()
        cv = args.chunk // 4
        nch = (V + cv - 1) // cv
        prev = S.current.clone()
        kern, algs, modes, k = [], [], [], 0
        dirty = None
        front = None   # vertices whose distance changed in the previous round (push frontier)
        while True:
            a, b = ev(), ev()
            i = S.k & 1
            a.record(st)
            _lib.check(rt.lib().proact_sssp_phase(S.gid, S.rid[i], S.rid[i ^ 1], int(S.k == 0), wl._s(st)), "sssp")
            b.record(st)
            rt.phase_sync(st, barrier=True)
            S.k += 1
            st.synchronize()
            kern.append(a.elapsed_time(b))
            mode = S.last_mode
            modes.append(mode)
            if mode == 0:   # pull (reading R13)
                de = S.e_own if dirty is None else int(epc[dirty].sum())
                algs.append(4.0 * S.e_own + 8.0 * de + 12.0 * (S.v1 - S.v0))
            else:           # push (reading R24): scan input + dprev, frontier out-edges, my vertices
                fe = int(outdeg[s0]) if front is None else int(outdeg[front].sum())
                algs.append(8.0 * V + 12.0 * fe + 12.0 * (S.v1 - S.v0))
            cur = S.current
            pad = nch * cv - V
            chg = cur != prev
            diff = torch.nn.functional.pad(chg.to(torch.int32), (0, pad))
            dirty = (diff.view(nch, cv).sum(1) > 0).cpu().numpy()
            front = chg.cpu().numpy()
            prev = cur.clone()
            k += 1
            if rt.last_vote() == 0 or k >= V:
                break
        out = {"rounds": rounds, "t": sum(times[args.warmup:]), "kern_ms": kern, "alg": algs, "modes": modes,
               "nhot": S.nhot, "e_own": S.e_own}
        if G == 1:   # tracking overhead: a whole run under ELIDE vs LOCAL
            oh = {}
            w0 = rt.get_config()["agent_warps"]
            for name, mech, aw in (("local", _lib.MECH_LOCAL, w0), ("elide", _lib.MECH_ELIDE, w0),
                                   ("local", _lib.MECH_LOCAL, w0), ("elide4", _lib.MECH_ELIDE, 4)):
                rt.set_config(mech=mech, agent_warps=aw)
                S.reset()
                t0 = time.perf_counter()
                S.run(stream=st)
                oh[name] = time.perf_counter() - t0
            oh["agent_warps"] = w0
            out["overhead"] = oh
            rt.set_config(agent_warps=w0, mech={v: k for k, v in _lib.MECH_NAMES.items()}[args.mech])
        S.free()
        return out
    epc = np.bincount(src // (args.chunk // 4), minlength=(V + args.chunk // 4 - 1) // (args.chunk // 4))
    outdeg = np.bincount(src, minlength=V)   # G = 1 roofline: every out-edge lands on this rank
    res = run_ranks(args.ranks, body)
    t = max(r["t"] for r in res)
    rounds = res[0]["rounds"]
    line = {"workload": f"sssp_rmat{args.scale}_ef16 (BASELINE.json config 4)",
            "value": args.steps * rounds / t, "unit": "rounds/s", "rounds": rounds, "ranks": args.ranks,
            "mech": args.mech, "chunk_bytes": args.chunk, "edges": int(src.size),
            "timing": "host wall clock per run (a BARRIER + host vote read every round)"}
    if "overhead" in res[0]:
        o = res[0]["overhead"]
        line["overhead"] = {"local_s_per_run": o["local"], "elide_s_per_run": o["elide"],
                            "tracking_overhead_frac": o["elide"] / o["local"] - 1.0,
                            "agent_warps": o["agent_warps"],
                            "tracking_overhead_frac_4_agent_warps": o["elide4"] / o["local"] - 1.0,
                            "note": "G=1: ELIDE keeps tallies + agent with remote stores skipped (Fig. 8 methodology)"}
    if args.ranks == 1:
        r0 = res[0]
        kms, alg = sum(r0["kern_ms"]), sum(r0["alg"])
        line["roofline"] = {"bound": "hbm", "kernel": ("sssp_hot_kernel" if r0["nhot"] else "sssp_kernel") + " / sssp_push_kernel",
                            "kernel_ms_per_round": [round(x, 4) for x in r0["kern_ms"]],
                            "mode_per_round": ["push" if m else "pull" for m in r0["modes"]],
                            "alg_bytes_per_run": alg, "achieved": alg / kms / 1e6, "peak": peak_hbm(),
                            "unit": "GB/s", "frac": alg / kms / 1e6 / peak_hbm(),
                            "note": "pull round: 4 B/in-edge scanned + 8 B/in-edge of a changed source chunk + 12 B/vertex; "
                                    "push round (R24): 8 B/vertex of the graph (input + previous input) + 12 B per "
                                    "frontier out-edge + 12 B/vertex of mine; summed over the run / summed kernel time"}
    if not args.no_cpu:
        import oracle
        tm = {}
        _, orounds, _ = oracle.sssp(V, src, dst, w, s0, timing=tm)   # to convergence, as the GPU run
        line["cpu_baseline"] = {"value": orounds / tm["iter_seconds"], "unit": "rounds/s",
                                "cores": oracle.get_threads(), "kind": "oracle",
                                "sample": f"oracle.sssp to convergence ({orounds} rounds) of the full graph on all "
                                          "host cores (OpenMP pull over in-edges); the CSC build is excluded"}
    return line


def micro(args):
    R = args.bytes
    W = R // 4

    def body(r, G):
        rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[args.mech])
        M = wl.Micro(W, args.chunk)
        s = torch.cuda.Stream()
        for _ in range(args.warmup):
            M.step(0x5EED, 1, False, stream=s, barrier=True)
        torch.cuda.synchronize()
        rt.host_barrier()
        e0, e1 = ev(), ev()
        e0.record(s)
        for _ in range(args.steps):
            M.step(0x5EED, 1, False, stream=s, barrier=True)
        e1.record(s)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1)
    ms = max(run_ranks(args.ranks, body))
    G = args.ranks
    repl = (G - 1) * R * args.steps   # bytes that cross "links" (to the G-1 other replicas)
    return {"workload": f"micro R={R} chunk={args.chunk} loopback G={G}", "value": repl / (ms / 1000.0) / 1e9,
            "unit": "GB/s replicated (HBM loopback)", "ms_per_phase": ms / args.steps, "mech": args.mech}


def banded(args):
    """NEXT-2: the paper's banded-matrix Jacobi (L271), N = 2^scale rows, half-bandwidth --w;
    step = 20 phases; roofline = (2w+1) x 4 B of A + 12 B (b, x read, x' write) per row / HBM."""
    N, w, I = 1 << args.scale, args.w, 20
    a, b = synth.banded(N, w)

    def body(r, G):
        rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[args.mech])
        B = wl.Banded(a, b, args.chunk)
        s = torch.cuda.Stream()
        for _ in range(2):
            B.step(s)
        torch.cuda.synchronize()
        rt.host_barrier()
        e0, e1 = ev(), ev()
        e0.record(s)
        for k in range(args.steps * I):
            B.step(s, barrier=(k == args.steps * I - 1))
        e1.record(s)
        torch.cuda.synchronize()
        ks = []
        for _ in range(10):
            x0, x1 = ev(), ev()
            i = B.k & 1
            x0.record(s)
            _lib.check(rt.lib().proact_banded_phase(B.rid[i], B.rid[i ^ 1], ctypes.c_void_p(B.a.data_ptr()),
                                                    ctypes.c_void_p(B.b.data_ptr()), B.N, B.w, wl._s(s)), "banded")
            x1.record(s)
            rt.phase_sync(s)
            B.k += 1
            ks.append((x0, x1))
        torch.cuda.synchronize()
        return {"ms": e0.elapsed_time(e1), "kms": statistics.median(x.elapsed_time(y) for x, y in ks),
                "rows": B.r1 - B.r0}
    res = run_ranks(args.ranks, body)
    ms = max(r["ms"] for r in res)
    kms = max(r["kms"] for r in res)
    alg = max(((2 * w + 1) * 4 + 12) * r["rows"] for r in res)
    line = {"workload": f"banded_jacobi N=2^{args.scale} w={w} (NEXT-2, PAPER.md L271)",
            "value": args.steps * I / (ms / 1000.0), "unit": "iters/s", "ranks": args.ranks, "mech": args.mech,
            "roofline": {"bound": "hbm",
                         "kernel": "banded_kernel" if (w > 4096 or os.environ.get("PROACT_BANDED_PLAIN", "0") != "0")
                         else "banded_tma_kernel", "kernel_ms": kms, "alg_bytes_per_launch": alg,
                         "achieved": alg / kms / 1e6, "peak": peak_hbm(), "unit": "GB/s",
                         "frac": alg / kms / 1e6 / peak_hbm(), "frac_spec_8000": alg / kms / 1e6 / 8000.0,
                         "note": "A is read once per sweep (97 % of the bytes are reads); the measured peak is a "
                                 "read+write copy figure, so a read stream can exceed it"}}
    if not args.no_cpu:
        import oracle
        t0 = time.perf_counter()
        oracle.banded_jacobi(a, b, np.zeros(N, dtype=np.float32), 2)
        dt = time.perf_counter() - t0
        line["cpu_baseline"] = {"value": 2 / dt, "unit": "iters/s", "cores": oracle.get_threads(), "kind": "oracle",
                                "sample": "2 oracle.banded_jacobi iterations"}
    return line


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="pagerank", choices=["pagerank", "sssp", "micro", "banded"])
    ap.add_argument("--w", type=int, default=16, help="banded: half-bandwidth")
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--chunk", type=int, default=128 * 1024)
    ap.add_argument("--mech", default="fused")
    ap.add_argument("--ranks", type=int, default=1)
    ap.add_argument("--bytes", type=int, default=256 << 20)
    ap.add_argument("--no-cpu", action="store_true")
    args = ap.parse_args()
    if args.workload in ("micro", "banded"):
        print(json.dumps(micro(args) if args.workload == "micro" else banded(args)), flush=True)
        return
    t0 = time.perf_counter()
    src, dst = synth.rmat(args.scale, 16)
    V = 1 << args.scale
    gen_s = time.perf_counter() - t0
    line = pagerank(args, src, dst, V) if args.workload == "pagerank" else sssp(args, src, dst, V)
    line["rmat_gen_s"] = gen_s
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
