#!/usr/bin/env python
"""bench.py -- PROACT hot path on B200: BASELINE.json's metric on config 2 (Jacobi 16384^2).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl proact|reference]
                    [--mech fused|inline|bulk|local|elide] [--chunk BYTES] [--iters I]

One STEP = one full solve of BASELINE.json config 2: I = 100 Jacobi phases of the
16384 x 16384 fp32 grid, rows strong-scaled over the N ranks, each phase = producer
kernel with fused transfer agent (tracking, polling, pushes, arrival flags) + phase
sync (credits).  value = iterations/s of the whole job (K*I / max-over-ranks time).
The grid (1 GiB per buffer) is far larger than L2 (126 MB), so no flush is needed.

Extra keys: roofline (dominant kernel = jacobi_kernel, HBM bound, measured live with
CUDA events on its stream), cpu_baseline (the oracle, rank 0, bounded sample), e2e
(proact_jacobi_solve_host with pinned host buffers: H2D of the grid + I phases + D2H),
clocks (nvidia-smi sampled during the timed region), gpu_launches, overhead (the
same step with the uninstrumented LOCAL mechanism: the paper's tracking-overhead
decomposition, Sec. V-C).  N = 1 also adds `secondary` (outside the timed
region): config 2 on two loopback ranks of this GPU with every transfer mechanism (the
PROACT path itself; at G = 1 nothing is replicated) and BASELINE.json configs 3-4
(PageRank / SSSP, RMAT-24) with their rooflines and oracle baselines, and a config-5
chunk sweep (transfer microbenchmark, the paper's Fig. 6 shape) on two loopback ranks.

--impl reference: the CPU oracle (oracle/) timed as it stands on the host cores, on
the same config/metric; rank 0 only under torchrun.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
# before torch touches CUDA: the agent kernel runs on its own high-priority stream, and with the
# default 8 hardware connections its launches can queue behind the producer stream's work
# (false dependencies: +100 us per phase measured, tools/probes/host_issue.py)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

METRIC = "strong-scaling speedup and iters/sec at 1/2/4/8 B200; NVLink GB/s vs 900 GB/s"
N_GRID = 16384
ITERS = 100
WORKLOAD = "jacobi2d_5pt_fp32_16384x16384_100it (BASELINE.json config 2, full replication)"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback"


def _sustained_copy_gbs(stream, seconds: float) -> dict:
    """torch copy_ of 1 Gi bf16 elements (MEASURED_PEAKS.json's recipe: read + write bytes) back to
    back for `seconds`, per-launch CUDA events; the median of the second half is the sustained
    copy bandwidth.  Calibration only: outside the timed region, not one of our kernels."""
    import torch
    n = 1 << 30
    a = torch.empty(n, dtype=torch.bfloat16, device="cuda")
    b = torch.empty_like(a)
    a.fill_(1.0)
    with torch.cuda.stream(stream):
        b.copy_(a)
        torch.cuda.synchronize()
        per = 4.0 * n / 6.4e12                     # rough seconds per copy, sizes the run
        reps = max(8, int(seconds / per))
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
        for e0, e1 in ev:
            e0.record(stream)
            b.copy_(a)
            e1.record(stream)
        torch.cuda.synchronize()
    t = [e0.elapsed_time(e1) for e0, e1 in ev]
    burst = min(t)
    late = statistics.median(t[reps // 2:])
    del a, b
    torch.cuda.empty_cache()
    return {"gbs": 4.0 * n / (late * 1e-3) / 1e9, "burst_gbs": 4.0 * n / (burst * 1e-3) / 1e9,
            "launches": reps, "note": "median of the second half of back-to-back 1 Gi bf16 copies, "
                                      "same recipe as MEASURED_PEAKS.json hbm_gbs; context, not the peak"}


def _traffic_from_profiles():
    """dram bytes per launch of jacobi_kernel from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_jacobi_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get("dram_bytes_per_launch")
    except Exception:
        return None


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = f"/tmp/proact_clocks_{os.getpid()}.csv"

    def __enter__(self):
        if self.index < 0:   # sampling disabled (diagnostics only)
            return self
        try:
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(5)
            except Exception:
                self.proc.kill()
            self.f.close()

    def summary(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        try:
            os.remove(self.path)
        except OSError:
            pass
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def max_over_ranks(ms: float, world: int) -> float:
    """Max of a per-rank time over all ranks (the contract's whole-job time); works with the
    nccl (CUDA tensor) and gloo (CPU tensor) backends."""
    if world <= 1:
        return float(ms)
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([float(ms)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def cpu_baseline(N: int, budget_s: float = 12.0) -> dict:
    """The oracle as it stands (oracle.jacobi_step, OpenMP over all host cores) on the full
    16384^2 grid, iterated until ~budget_s of CPU work (bounded sample)."""
    import numpy as np
    import oracle
    import synth
    x = synth.jacobi_init(N)
    oracle.jacobi_step(x)   # page in / warm
    t0 = time.perf_counter()
    k = 0
    while True:
        x = oracle.jacobi_step(x)
        k += 1
        if time.perf_counter() - t0 > budget_s or k >= ITERS:
            break
    dt = time.perf_counter() - t0
    del np
    return {"value": k / dt, "unit": "iters/s", "cores": oracle.get_threads(), "kind": "oracle",
            "sample": f"{k} Jacobi iterations of the full {N}x{N} fp32 grid (oracle.jacobi_step)"}


def single_gpu_reference(N: int, I: int, rpt: int, steps: int = 2) -> float:
    """Milliseconds for `steps` uninstrumented single-GPU solves (G = 1, LOCAL: the plain
    producer kernel) of the full grid on this rank's GPU: the strong-scaling denominator,
    measured in the same run, before the N-rank context exists (its own one-rank context)."""
    import torch
    import synth
    from paper_conf_isca_muthukrishnannl21_b200 import _lib
    from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
    from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl
    rt.init(1, 0, rt.new_job_key())
    rt.set_config(mech=_lib.MECH_LOCAL)
    J = wl.Jacobi(N, 1 << 20, x0=torch.from_numpy(synth.jacobi_init(N)).cuda(), rows_per_tile=rpt)
    s = torch.cuda.Stream()
    for k in range(I):
        J.step(s, barrier=(k == I - 1))
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.synchronize()
    a.record(s)
    for _ in range(steps):
        for k in range(I):
            J.step(s, barrier=(k == I - 1))
    b.record(s)
    s.synchronize()
    ms = a.elapsed_time(b)
    rt.check_device()
    del J
    torch.cuda.synchronize()
    rt.finalize()
    torch.cuda.empty_cache()
    return ms


def _json_lines(cmd: list, env: dict, timeout: float) -> list:
    """Run a helper (tools/) in its own process; its stdout JSON lines, or an error record."""
    try:
        r = subprocess.run(cmd, env=env, cwd=ROOT, capture_output=True, text=True, timeout=timeout)
    except subprocess.TimeoutExpired:
        return [{"error": f"timeout after {timeout:.0f}s"}]
    out = []
    for line in r.stdout.splitlines():
        line = line.strip()
        if line.startswith("{"):
            try:
                out.append(json.loads(line))
            except ValueError:
                pass
    if r.returncode != 0 or not out:
        out.append({"error": f"rc={r.returncode}: {r.stderr.strip().splitlines()[-1:] if r.stderr else ''}"})
    return out


def secondary_legs(N: int, peak: float) -> dict:
    """N = 1 only, after the headline's context is finalised and its memory freed (nothing here is
    inside the timed region).  At G = 1 nothing is replicated (reading R18), so the PROACT
    transfer path is measured here on this one GPU the only way it can be: two ranks as threads
    ("loopback") of config 2, every mechanism on the same ranks -- the replica
    bytes cross HBM, not NVLink, so these rank the mechanisms on this box; they are not NVLink
    numbers.  Also BASELINE.json configs 3 and 4 (PageRank / SSSP on RMAT-24) with their own
    roofline and oracle baseline (tools/bench_workloads.py)."""
    py = sys.executable
    env = dict(os.environ)
    env.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
    names = {("fused", 2): "proact_producer_tile_push", ("fused", 1): "proact_separate_agent",
             ("fused", 0): "proact_agent_in_grid", ("elide", 2): "elide_tracking_only_tile_push",
             ("elide", 1): "elide_tracking_only_separate_agent", ("inline", None): "naive_p2p_inline",
             ("bulk", None): "bulk_cudaMemcpyPeer", ("dma", None): "dma_copy_engine_program",
             ("local", None): "local_no_transfer"}
    legs = {
        "full": dict(HALO="0", CHUNKS="1048576", MECHS="fused,elide,inline,bulk,dma,local", AKERNS="2,1",
                     PUSHES="1", WARPS="32"),
        "halo_only": dict(HALO="1", CHUNKS="131072", MECHS="fused,inline,bulk,dma,local", AKERNS="1,2",
                          PUSHES="0", WARPS="2"),
    }
    gib = float(1 << 30)
    # loopback HBM floor per phase (whole device): both ranks' stencil traffic (8 B/cell of the
    # grid) + the replicated half each rank writes into the other's replica (4 B/cell), full
    # replication; halo-only adds two rows
    floor_bytes = {"full": 8.0 * N * N + 4.0 * N * N, "halo_only": 8.0 * N * N + 2 * 4.0 * N}
    out = {"note": ("G = 2 loopback ranks of config 2 on this one GPU (replica bytes cross HBM, not NVLink: "
                    "mechanism ranking on this box, not an NVLink result); ms per phase, max over ranks, "
                    "20 phases after 3 warm-up")}
    for leg, kv in legs.items():
        e = dict(env, G="2", N=str(N), PHASES="20", **kv)
        pts = _json_lines([py, os.path.join(ROOT, "tools", "sweep_jacobi_loop.py")], e, 600)
        ms = {}
        for p in pts:
            if "error" in p:
                ms.setdefault("errors", []).append(p["error"])
                continue
            key = (p["mech"], p["akern"] if p["mech"] in ("fused", "elide") else None)
            ms[names.get(key, f"{p['mech']}_{p['akern']}")] = p["ms"]
        proact = {k: v for k, v in ms.items() if k.startswith("proact_")}
        base = {k: ms[k] for k in ("naive_p2p_inline", "bulk_cudaMemcpyPeer", "dma_copy_engine_program") if k in ms}
        best = min(proact, key=proact.get) if proact else None
        out[leg] = {"ms_per_phase": ms, "chunk_bytes": int(kv["CHUNKS"]),
                    "hbm_floor_ms": floor_bytes[leg] / (peak * 1e9) * 1e3,
                    "best_proact": best,
                    "best_proact_vs_baselines": ({k: v / proact[best] for k, v in base.items()} if best else None)}
        if "local_no_transfer" in ms and "bulk_cudaMemcpyPeer" in ms and best:
            opp = ms["bulk_cudaMemcpyPeer"] - ms["local_no_transfer"]
            out[leg]["opportunity_captured"] = ((ms["bulk_cudaMemcpyPeer"] - proact[best]) / opp) if opp > 0 else None
            out[leg]["opportunity_note"] = ("(T_bulk - T_proact) / (T_bulk - T_local); above 1 = the PROACT phase ran "
                                            "faster than the no-transfer LOCAL phase on these ranks (run-to-run noise "
                                            "of a few us when the opportunity itself is a few us)")
    # config 5 (transfer microbenchmark, the paper's Fig. 6 shape): chunk sweep, PROACT (producer
    # placement) vs the baselines, two loopback ranks, R = 256 MiB, pure mode (K = 1)
    e = dict(env, G="2", RBYTES=str(256 << 20), K="1", CHUNKS="4096,65536,1048576,4194304",
             MECHS="fused,inline,bulk,dma", AKERNS="2", PUSHES="1", WARPS="8", PHASES="8")
    pts = _json_lines([py, os.path.join(ROOT, "tools", "sweep_micro.py")], e, 600)
    fig6 = {}
    for p in pts:
        if "error" in p:
            fig6.setdefault("errors", []).append(p["error"])
            continue
        name = {"fused": "proact_producer_tile_push", "inline": "naive_p2p_inline", "bulk": "bulk_cudaMemcpyPeer",
                "dma": "dma_copy_engine_program"}.get(p["mech"], p["mech"])
        fig6.setdefault(str(p["chunk"]), {})[name] = p["ms"]
    for ch, row in fig6.items():
        if ch != "errors" and "proact_producer_tile_push" in row and "bulk_cudaMemcpyPeer" in row:
            row["speedup_vs_bulk"] = row["bulk_cudaMemcpyPeer"] / row["proact_producer_tile_push"]
    out["micro_fig6"] = {"ms_per_phase_by_chunk": fig6, "R_bytes": 256 << 20, "G": 2,
                         "note": "BASELINE.json config 5 shape (all-gather of R, pure mode), loopback"}
    for wk in ("pagerank", "sssp"):
        pts = _json_lines([py, os.path.join(ROOT, "tools", "bench_workloads.py"), "--workload", wk,
                           "--steps", "3", "--warmup", "1"], env, 900)
        out[wk] = pts[0] if len(pts) == 1 else pts
    return out


def run_reference(args, dist_rank: int) -> None:
    if dist_rank != 0:
        return
    N = args.n
    cb = cpu_baseline(N, budget_s=max(2.0, 60.0 / max(1, args.steps + args.warmup)))
    # each step: a bounded sample of the workload (cb's iterations), timed on the host
    import oracle
    import synth
    x = synth.jacobi_init(N)
    per = max(1, int(round(cb["value"] * 3.0)))   # ~3 s of oracle work per step
    for _ in range(args.warmup):
        x = oracle.jacobi_step(x)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        for _ in range(per):
            x = oracle.jacobi_step(x)
    dt = time.perf_counter() - t0
    v = args.steps * per / dt
    cbr = dict(cb)
    cbr["value"] = v
    cbr["sample"] = f"{args.steps} steps x {per} oracle Jacobi iterations of the {N}x{N} grid"
    line = {"metric": METRIC, "value": v, "unit": "iters/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1000.0 * dt / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "impl": "reference", "config": {"workload": WORKLOAD, "N": N, "iters_per_step": per},
            "cpu_baseline": cbr, "e2e": {"value": v, "unit": "iters/s", "h2d_bytes_per_step": 0,
                                         "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)   # >= 3 nvidia-smi samples (100 ms) in the timed region
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="proact", choices=["proact", "reference"])
    ap.add_argument("--mech", default="fused")
    ap.add_argument("--chunk", type=int, default=0)
    ap.add_argument("--warps", type=int, default=0)
    ap.add_argument("--rpt", type=int, default=32)   # sustained-load sweep r01v: 32 > 64 > 16 > 8
    ap.add_argument("--iters", type=int, default=ITERS)
    ap.add_argument("--grid-n", dest="n", type=int, default=N_GRID)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-baselines", action="store_true", help="N > 1: skip the bulk / inline / NCCL legs")
    ap.add_argument("--no-tune", action="store_true", help="N > 1: keep the default chunk / agent warps")
    ap.add_argument("--no-overhead", action="store_true",
                    help="skip the ELIDE tracking-overhead leg (its agent kernel must run concurrently "
                         "with the producer, which a kernel-serialising profiler prevents)")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for the timing barrier / max-over-ranks only")
    ap.add_argument("--no-halo", action="store_true", help="N > 1: skip the halo-only legs")
    ap.add_argument("--no-n1", action="store_true", help="N > 1: skip the single-GPU reference (speedup)")
    ap.add_argument("--no-secondary", action="store_true",
                    help="N = 1: skip the loopback mechanism legs and the PageRank / SSSP configs")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank)
        return
    # the oracle baseline first, before this process pins host memory or touches the GPU (a
    # later run shared the host with 2 GiB of pinned e2e buffers and measured ~3x slower)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(args.n)

    import torch
    import torch.distributed as dist
    from paper_conf_isca_muthukrishnannl21_b200 import _lib
    from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
    from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl
    import synth

    # PROACT_BENCH_SAME_DEVICE=1: every rank on GPU 0 (tests of the multi-process path on a
    # one-GPU box; ranks then time-slice, so such numbers are not performance)
    dev = 0 if os.environ.get("PROACT_BENCH_SAME_DEVICE") == "1" else local
    torch.cuda.set_device(dev)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group("gloo")
        job = f"bench_{os.environ.get('MASTER_ADDR', '')}_{os.environ.get('MASTER_PORT', '')}"
    else:
        job = rt.new_job_key()
    # strong-scaling denominator: the uninstrumented single-GPU solve, on every rank's GPU at once
    n1_ms = None
    if world > 1 and not args.no_n1:
        n1_ms = max_over_ranks(single_gpu_reference(args.n, args.iters, args.rpt), world)
    rt.init(world, rank, job)
    # --mech nccl: the north star's bulk baseline -- uninstrumented kernels (LOCAL) with an NCCL
    # all-gather of the rows between them (workloads.Jacobi.step_allgather)
    nccl_base = args.mech == "nccl"
    mode = {"nccl": nccl_base}
    mech = _lib.MECH_LOCAL if nccl_base else {v: k for k, v in _lib.MECH_NAMES.items()}[args.mech]
    cfg = rt.get_config()
    chunk = args.chunk or cfg["chunk_bytes"]
    kw = {"mech": mech}
    if args.warps:
        kw["agent_warps"] = args.warps
    cfg = rt.set_config(**kw)
    N, I = args.n, args.iters
    x0 = torch.from_numpy(synth.jacobi_init(N)).cuda()
    # NVLS: on an NVSwitch system with every rank a thread of one process... (torchrun ranks are
    # processes, so proact_mcast_supported() is 0 there and the replicas are plain tensors)
    mcast = world > 1 and rt.mcast_supported()
    J = wl.Jacobi(N, chunk, x0=x0, rows_per_tile=args.rpt, mcast=mcast)
    del x0
    s = torch.cuda.Stream()

    # N > 1, PROACT mechanism, no explicit --warps/--chunk: the paper's profiler (Sec. III-A,
    # a9) picks chunk size and agent warps for this G before anything is timed -- the transfer
    # volume grows with G - 1, so one fixed agent size cannot fit 2 and 8 GPUs.  A small space
    # (3 warm + 5 timed phases per point, max over ranks), a fresh cache file per job.
    tuned = None
    if world > 1 and args.mech == "fused" and not args.warps and not args.chunk and not args.no_tune:
        os.environ["PROACT_TUNE_CACHE"] = f"/tmp/proact_tune_{job}.json"

        def run_point(c):
            if c["chunk_bytes"] != rt.region_info(J.rid[0]).chunk_bytes:
                for rid in J.rid:
                    rt.rechunk(rid, c["chunk_bytes"])
            for _ in range(3):
                J.step(s)
            ts = []
            for _ in range(5):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                J.step(s, barrier=True)
                b.record(s)
                s.synchronize()
                ts.append(a.elapsed_time(b))
            return statistics.median(ts)

        space = "mech=0;chunk=131072,1048576;warps=8,16,32;push=0,1" + (",2" if mcast else "") + ";akern=0,1,2"
        best = rt.autotune(f"bench_jacobi_N{N}_G{world}", run_point, space)
        if best["chunk_bytes"] != rt.region_info(J.rid[0]).chunk_bytes:
            for rid in J.rid:
                rt.rechunk(rid, best["chunk_bytes"])
        cfg = rt.set_config(mech=best["mech"], agent_warps=best["agent_warps"], push=best["push"],
                            agent_kernel=best["agent_kernel"], chunk_bytes=best["chunk_bytes"])
        chunk = best["chunk_bytes"]
        tuned = {"space": space, "best": {k: best[k] for k in ("chunk_bytes", "agent_warps", "push", "agent_kernel")},
                 "note": "proact_autotune (a9): chunk x agent warps x push (VEC16 / TMA) x agent placement "
                         "(fused CTAs / separate kernel / producer-CTA transfer warps); max over ranks"}

    live_ev: list = []   # (start, end) CUDA event pairs around jacobi_kernel inside the timed region

    def step():
        if mode["nccl"]:
            for k in range(I):
                J.step_allgather(s)
            return
        if mode.get("live") is None:
            for k in range(I):
                J.step(s, barrier=(k == I - 1))
            return
        # same launches as J.step, with the producer kernel bracketed by events on its stream
        pool = mode["live"]
        for k in range(I):
            a, b = pool.pop()
            i = J.k & 1
            a.record(s)
            wl.jacobi_phase(J.rid[i], J.rid[i ^ 1], N, J.rpt, s)
            b.record(s)
            rt.phase_sync(s, barrier=(k == I - 1))
            J.k += 1
            live_ev.append((a, b))

    per_step: list = []   # this rank's per-step times of the last timed() call (spread check)

    def timed(fn, K):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(K + 1)]
        ev[0].record(s)
        for k in range(K):
            fn()
            ev[k + 1].record(s)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        per_step.clear()
        per_step.extend(ev[k].elapsed_time(ev[k + 1]) for k in range(K))
        return max_over_ranks(ev[0].elapsed_time(ev[K]), world)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    l0 = rt.launch_count()
    if not mode["nccl"]:
        mode["live"] = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                        for _ in range(args.steps * I)]
    with Clocks(dev if os.environ.get("PROACT_BENCH_NO_CLOCKS") != "1" else -1) as clk:
        ms = timed(step, args.steps)
    mode["live"] = None
    step_ms = list(per_step)
    launches = rt.launch_count() - l0
    rt.check_device()
    value = args.steps * I / (ms / 1000.0)

    # ---- roofline of the dominant kernel: per-launch CUDA events around jacobi_kernel, recorded
    # live inside the timed region (kms); a short isolated run after it is kept for context
    evs = []
    for k in range(2 * 10):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        i = J.k & 1
        a.record(s)
        wl.jacobi_phase(J.rid[i], J.rid[i ^ 1], N, J.rpt, s)
        b.record(s)
        rt.phase_sync(s, barrier=False)
        J.k += 1
        evs.append((a, b))
    torch.cuda.synchronize()
    kms_isolated = statistics.mean(a.elapsed_time(b) for a, b in evs)
    live_t = [a.elapsed_time(b) for a, b in live_ev]
    kms = statistics.mean(live_t) if live_t else kms_isolated
    live_trend = ([statistics.median(live_t[:max(1, len(live_t) // 10)]),
                   statistics.median(live_t[len(live_t) // 2:])] if live_t else None)
    nrows = J.r1 - J.r0
    alg_bytes = 8.0 * N * nrows          # read x^k + write x^{k+1} of my rows
    peaks, src = _peaks()
    peak = float(peaks.get("hbm_gbs", 6650.0))
    achieved = alg_bytes / (kms / 1000.0) / 1e9
    # whole-phase roofline of SURVEY.md Sec. 8(d): T_roof = max(T_HBM, T_NVL) per rank, T_HBM =
    # my rows' 8 B/cell at the HBM peak, T_NVL = the replicated ingress ((G-1)/G of the grid,
    # full replication) at 900 GB/s per direction; frac = T_roof / measured phase time
    NVL = 900.0
    ingress = 4.0 * N * (N - nrows)      # bytes pushed INTO this rank per phase (max over ranks ~ equal)
    t_phase_us = ms / (args.steps * I) * 1000.0
    t_hbm_us = alg_bytes / (peak * 1e9) * 1e6
    t_nvl_us = ingress / (NVL * 1e9) * 1e6
    step_roofline = {"t_hbm_us": t_hbm_us, "t_nvl_us": t_nvl_us, "t_phase_us": t_phase_us,
                     "frac": max(t_hbm_us, t_nvl_us) / t_phase_us,
                     "nvlink_ingress_GBps_per_gpu": ingress / (t_phase_us * 1e-6) / 1e9, "nvlink_peak_GBps": NVL,
                     "note": "per rank and phase; NVLink 900 GB/s/direction nominal (B200_PROFILING.md)"}
    # context for the live fraction: the MEASURED_PEAKS.json copy recipe (1 Gi bf16 elements,
    # read + write bytes) run back to back for about as long as the timed region, on this box, now
    sustained = None
    if os.environ.get("PROACT_BENCH_NO_SUSTAINED") != "1":
        sustained = _sustained_copy_gbs(s, max(0.1, ms / 1000.0))
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": _traffic_from_profiles(),
                "kernel": "jacobi_kernel", "kernel_ms": kms, "alg_bytes_per_launch": alg_bytes,
                "kernel_ms_source": ("mean of %d launches timed live in the timed region" % len(live_ev)
                                     if live_ev else "isolated 20-launch run"),
                "kernel_ms_isolated": kms_isolated,
                "kernel_ms_live_first10pct_last50pct": live_trend,
                "sustained_copy": sustained,
                "frac_of_sustained_copy": (achieved / sustained["gbs"]) if sustained else None,
                "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({src})"}

    # ---- tracking overhead (Sec. V-C, Fig. 8): the same step with
    # instrumentation + agent but no remote stores (ELIDE) vs the uninstrumented kernel (LOCAL)
    overhead = None
    if world == 1 and not args.no_overhead:
        kk = max(2, args.steps // 2)
        res = {}
        for name, m in (("local", _lib.MECH_LOCAL), ("elide", _lib.MECH_ELIDE)):
            rt.set_config(mech=m)
            step()
            res[name] = kk * I / (timed(step, kk) / 1000.0)
        overhead = {"local_iters_per_s": res["local"], "elide_iters_per_s": res["elide"],
                    "tracking_overhead_frac": res["local"] / res["elide"] - 1.0,
                    "note": "G=1: FUSED has nothing to send and runs the LOCAL kernel; ELIDE keeps "
                            "tallies + agent (paper's instrumentation-only run)"}
        rt.set_config(mech=mech)

    # ---- baselines on the same ranks (north star: beat bulk DMA / NCCL all-gather and naive
    # P2P stores): iterations/s of the same step with each mechanism, N > 1 only (at N = 1
    # there is nothing to move and every mechanism is the plain kernel)
    baselines = None
    try:   # an optional leg: a failure is reported in the line, not fatal to it
        if world > 1 and not args.no_baselines:
            baselines = {}
            kk = max(2, args.steps // 2)
            legs = [("bulk_cudaMemcpyPeer", _lib.MECH_BULK, False), ("naive_p2p_inline", _lib.MECH_INLINE, False)]
            if dist.get_backend() == "nccl":
                legs.append(("nccl_allgather", _lib.MECH_LOCAL, True))
            for name, m, use_nccl in legs:
                rt.set_config(mech=m)
                mode["nccl"] = use_nccl
                step()
                baselines[name] = kk * I / (timed(step, kk) / 1000.0)
            mode["nccl"] = nccl_base
            rt.set_config(mech=mech)
    except Exception as ex:   # noqa: BLE001
        baselines = {"error": f"{type(ex).__name__}: {ex}"[:300]}
        mode["nccl"] = nccl_base
        try:
            rt.set_config(mech=mech)
        except Exception:   # noqa: BLE001
            pass

    # ---- NEXT-1, the paper's decomposition (Sec. V-C; Fig. 8/9) on the same
    # ranks: LOCAL = no transfer at all and no waits (the infinite-bandwidth bound; replicas go
    # stale, timing only), ELIDE = tracking + agent without remote stores (tracking overhead), BULK
    # = transfers after the kernel.  opportunity = T_bulk - T_local; captured = (T_bulk - T_proact)
    # / opportunity; overlap = captured with the tracking overhead added back
    decomposition = None
    try:   # an optional leg: a failure is reported in the line, not fatal to it
        if world > 1 and not args.no_baselines and baselines and mech in (_lib.MECH_FUSED, _lib.MECH_ELIDE):
            kk = max(2, args.steps // 2)
            dv = {}
            for name, m in (("local", _lib.MECH_LOCAL), ("elide", _lib.MECH_ELIDE)):
                rt.set_config(mech=m)
                step()
                dv[name] = timed(step, kk) / (kk * I)   # ms per phase
            rt.set_config(mech=mech)
            t_p = ms / (args.steps * I)
            t_b = 1000.0 / baselines["bulk_cudaMemcpyPeer"]
            opp = t_b - dv["local"]
            decomposition = {"ms_per_phase": {"proact": t_p, "bulk": t_b, "local_no_transfer": dv["local"],
                                              "elide_tracking_only": dv["elide"]},
                             "tracking_overhead_frac": dv["elide"] / dv["local"] - 1.0,
                             "opportunity_ms": opp,
                             "opportunity_captured": (t_b - t_p) / opp if opp > 0 else None,
                             "overlap_frac": (t_b - t_p + dv["elide"] - dv["local"]) / opp if opp > 0 else None,
                             "note": "paper Sec. V-C: infinite-BW bound = LOCAL, tracking overhead = ELIDE vs LOCAL"}
    except Exception as ex:   # noqa: BLE001
        decomposition = {"error": f"{type(ex).__name__}: {ex}"[:300]}
        mode["nccl"] = nccl_base
        try:
            rt.set_config(mech=mech)
        except Exception:   # noqa: BLE001
            pass

    # ---- halo-only variant (reading R8: the one config-2 variant whose roofline allows
    # >= 6x at G = 8): per-chunk destinations = the neighbours; PROACT (tuned) and the baselines
    halo = None
    try:   # an optional leg: a failure is reported in the line, not fatal to it
        if world > 1 and not args.no_halo:
            J.set_halo_only()
            kk = max(2, args.steps // 2)
            # the halo exchange moves two rows per rank: the profiler picks again, over few agent warps
            # (chunks bound nowhere never reach the agent) and the producer-CTA placement
            full_cfg = rt.get_config()
            halo_tuned = None
            if tuned is not None:
                def run_halo(c):
                    if c["chunk_bytes"] != rt.region_info(J.rid[0]).chunk_bytes:
                        for rid in J.rid:
                            rt.rechunk(rid, c["chunk_bytes"])
                        J.set_halo_only()   # rechunk drops per-chunk destinations
                    for _ in range(3):
                        J.step(s)
                    ts = []
                    for _ in range(5):
                        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        a.record(s)
                        J.step(s, barrier=True)
                        b.record(s)
                        s.synchronize()
                        ts.append(a.elapsed_time(b))
                    return statistics.median(ts)

                hspace = "mech=0;chunk=131072,1048576;warps=1,2,4;push=0,1;akern=0,1,2"
                hb = rt.autotune(f"bench_jacobi_halo_N{N}_G{world}", run_halo, hspace)
                if hb["chunk_bytes"] != rt.region_info(J.rid[0]).chunk_bytes:
                    for rid in J.rid:
                        rt.rechunk(rid, hb["chunk_bytes"])
                    J.set_halo_only()
                rt.set_config(agent_warps=hb["agent_warps"], push=hb["push"], agent_kernel=hb["agent_kernel"])
                halo_tuned = {"space": hspace, "best": {k: hb[k] for k in ("chunk_bytes", "agent_warps", "push",
                                                                         "agent_kernel")}}
            legs = [("proact", mech), ("bulk_cudaMemcpyPeer", _lib.MECH_BULK), ("naive_p2p_inline", _lib.MECH_INLINE)]
            hv = {}
            for name, m in legs:
                rt.set_config(mech=m)
                mode["nccl"] = False
                step()
                hv[name] = kk * I / (timed(step, kk) / 1000.0)
            mode["nccl"] = nccl_base
            rt.set_config(mech=mech, agent_warps=full_cfg["agent_warps"], push=full_cfg["push"],
                          agent_kernel=full_cfg["agent_kernel"])
            h_rows = (1 if rank > 0 else 0) + (1 if rank < world - 1 else 0)
            h_ingress = 4.0 * N * max(1, h_rows) if world > 1 else 0.0
            ht = 1000.0 / hv["proact"] * 1000.0   # us per phase
            h_nvl = h_ingress / (NVL * 1e9) * 1e6
            halo = {"value": hv["proact"], "unit": "iters/s", "tuned": halo_tuned,
                    "baselines_iters_per_s": {k: v for k, v in hv.items() if k != "proact"},
                    "speedup_vs_n1": None,
                    "step_roofline": {"t_hbm_us": t_hbm_us, "t_nvl_us": h_nvl, "t_phase_us": ht,
                                      "frac": max(t_hbm_us, h_nvl) / ht,
                                      "nvlink_ingress_GBps_per_gpu": h_ingress / (ht * 1e-6) / 1e9},
                    "note": "per-chunk destinations = neighbours (boundary rows only); rows other ranks own "
                            "are not replicated"}
    except Exception as ex:   # noqa: BLE001
        halo = {"error": f"{type(ex).__name__}: {ex}"[:300]}
        mode["nccl"] = nccl_base
        try:
            rt.set_config(mech=mech)
        except Exception:   # noqa: BLE001
            pass

    n1_value = (2 * I / (n1_ms / 1000.0)) if n1_ms else (value if world == 1 else None)
    if halo is not None and n1_value and "value" in halo:
        halo["speedup_vs_n1"] = halo["value"] / n1_value
    # transfer-agent cost: SMs dedicated to the agent x phase time per GB pushed
    egress_gb = 4.0 * N * nrows * (world - 1) / 1e9
    akern = cfg.get("agent_kernel", 1)
    agent_sms = 0 if akern == _lib.AGENT_PRODUCER else min(cfg["agent_warps"], 148 // 2)
    agent_cost = None
    if world > 1 and egress_gb > 0 and mech in (_lib.MECH_FUSED, _lib.MECH_ELIDE):
        agent_cost = {"agent_placement": {0: "fused CTAs", 1: "separate kernel", 2: "producer-CTA transfer warps"}[akern],
                      "dedicated_sms": agent_sms,
                      "agent_sm_ms_per_GB_pushed": agent_sms * (t_phase_us / 1000.0) / egress_gb,
                      "egress_GB_per_phase": egress_gb}

    # ---- e2e through the C-ABI host-buffer entry point
    e2e = None
    try:   # an optional leg: a failure is reported in the line, not fatal to it
        if not args.no_e2e:
            xh = torch.from_numpy(synth.jacobi_init(N)).pin_memory()
            out = torch.empty((N, N), dtype=torch.float32).pin_memory()
            nb = [0, 0]

            def e2e_step():
                h, d = wl.jacobi_solve_host(xh, out, N, I, chunk, args.rpt, s)
                nb[0], nb[1] = h, d

            e2e_step()
            torch.cuda.synchronize()
            ems = timed(e2e_step, max(2, min(args.steps, 3)))
            seq = max(2, min(args.steps, 3)) * I / (ems / 1000.0)
            # the pipelined entry point: K solves (steps), each with its own H2D of the input and D2H
            # of its result inside the timed region, solve k's phases overlapping the copies of k +- 1
            outs = [out, torch.empty((N, N), dtype=torch.float32).pin_memory()]
            # a stream of K solves: the first H2D and the last D2H (each ~19 ms over PCIe, measured
            # full duplex by tools/probes/pcie_duplex.py) cannot overlap compute; K amortises them
            K = max(4, min(2 * args.steps, 20))

            def e2e_pipe(k):
                h, d = wl.jacobi_solve_host_pipelined(xh, [outs[j & 1] for j in range(k)], N, I, chunk, args.rpt, s)
                nb[0], nb[1] = h, d

            e2e_pipe(2)
            torch.cuda.synchronize()
            pms = timed(lambda: e2e_pipe(K), 1)
            e2e = {"value": K * I / (pms / 1000.0), "unit": "iters/s",
                   "h2d_bytes_per_step": nb[0], "d2h_bytes_per_step": nb[1],
                   "api": "proact_jacobi_solve_host_pipelined", "steps": K,
                   "sequential_value": seq, "sequential_api": "proact_jacobi_solve_host"}
            del xh, out, outs   # 3 GiB of pinned host memory: release before the secondary legs
    except Exception as ex:   # noqa: BLE001
        e2e = {"error": f"{type(ex).__name__}: {ex}"[:300]}
        mode["nccl"] = nccl_base
        try:
            rt.set_config(mech=mech)
        except Exception:   # noqa: BLE001
            pass

    line = None
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "iters/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
                "dtype": "f32", "data": "synthetic",
                "config": {"workload": WORKLOAD, "N": N, "iters_per_step": I, "ranks": world,
                           "mech": args.mech,
                           "mech_effective": ("local (G = 1: nothing to replicate, so FUSED runs the "
                                              "uninstrumented kernel, reading R18)"
                                              if world == 1 and args.mech == "fused" else args.mech),
                           "chunk_bytes": chunk,
                           "agent_warps": cfg["agent_warps"], "piece_bytes": cfg["piece_bytes"],
                           "rows_per_tile": args.rpt, "replication": "full", "tuned": tuned, "nvls_multicast": mcast,
                           "l2": "inputs > L2 (two 1 GiB grids), no flush",
                           "parallelism": f"rows{world}",
                           "step_ms_min_median_max": [min(step_ms), statistics.median(step_ms), max(step_ms)]},
                "roofline": roofline, "step_roofline": step_roofline, "cpu_baseline": cpu, "e2e": e2e,
                "clocks": clk.summary(), "gpu_launches": launches, "overhead": overhead,
                "baselines_iters_per_s": baselines,
                "speedup_vs_n1": (value / n1_value) if n1_value else None,
                "n1_reference": {"value": n1_value, "unit": "iters/s",
                                 "what": ("this run's timed step (G = 1)" if world == 1 else
                                          "uninstrumented single-GPU solve (LOCAL) of the full grid on every "
                                          "rank's GPU in this run, slowest rank")},
                "halo_only": halo, "agent_cost": agent_cost, "decomposition": decomposition}
    torch.cuda.synchronize()
    J.free()
    del J
    rt.finalize()
    if world > 1:
        dist.destroy_process_group()
    if line is not None:
        if world == 1 and not args.no_secondary:
            torch.cuda.empty_cache()
            line["secondary"] = secondary_legs(N, peak)
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
