"""Loopback Jacobi sweep (config 2 shape, G ranks as threads on one GPU): per mechanism / agent
placement / push engine / agent warps / chunk, the time of a phase (producer + agent + sync),
max over ranks.  Replication bytes cross HBM here (no NVLink on a one-GPU box), and the ranks
split the device's SMs, so these numbers rank configurations; they are not NVLink results.

    G=2 N=16384 MECHS=fused,dma,bulk,inline AKERNS=0,1 PUSHES=0,1 WARPS=16 python tools/sweep_jacobi_loop.py
"""
import itertools
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # loopback ranks: see loopback.py
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

G = int(os.environ.get("G", 2))
N = int(os.environ.get("N", 16384))
HALO = os.environ.get("HALO", "0") == "1"
NODEST = os.environ.get("HALO", "0") == "2"   # diagnostics: every chunk bound nowhere
chunks = [int(x) for x in os.environ.get("CHUNKS", "131072").split(",")]
mechs = os.environ.get("MECHS", "fused,dma,bulk,inline").split(",")
warps = [int(x) for x in os.environ.get("WARPS", "16").split(",")]
pushes = [int(x) for x in os.environ.get("PUSHES", "1").split(",")]
akerns = [int(x) for x in os.environ.get("AKERNS", "0,1").split(",")]
PH = int(os.environ.get("PHASES", 10))
RPT = int(os.environ.get("RPT", 32))   # rows per tile (bench.py default)
x0 = synth.jacobi_init(N)


def body(r, G_):
    J = wl.Jacobi(N, chunks[0], x0=torch.from_numpy(x0).cuda(), halo_only=HALO, rows_per_tile=RPT)
    if NODEST:
        for rid in J.rid:
            for c in range(rt.region_info(rid).n_own_chunks):
                rt.set_chunk_dest(rid, c, 0)
    s = torch.cuda.Stream()
    out = []
    for ch in chunks:
        if ch != rt.region_info(J.rid[0]).chunk_bytes:
            for rid in J.rid:
                rt.rechunk(rid, ch)
            if HALO:
                J.set_halo_only()
        for mech, w, pu, ak in itertools.product(mechs, warps, pushes, akerns):
            if mech not in ("fused", "elide") and (w != warps[0] or pu != pushes[0] or ak != akerns[0]):
                continue
            if mech == "nccl":
                continue
            rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[mech], agent_warps=w, push=pu,
                          agent_kernel=ak)
            for _ in range(3):
                J.step(s, barrier=True)
            s.synchronize()
            rt.host_barrier()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            for k in range(PH):
                J.step(s, barrier=(k == PH - 1))
            b.record(s)
            s.synchronize()
            rt.host_barrier()
            out.append({"chunk": ch, "mech": mech, "warps": w, "push": pu, "akern": ak, "rpt": RPT,
                        "ms": a.elapsed_time(b) / PH})
    rt.check_device()
    return out


res = run_ranks(G, body)
for i, pt in enumerate(res[0]):
    ms = max(res[g][i]["ms"] for g in range(G))
    ingress = (G - 1) / G * N * N * 4 if not HALO else 2 * N * 4
    pt.update({"G": G, "N": N, "halo": HALO, "ms": ms, "ingress_GBps": ingress / ms / 1e6})
    print(json.dumps(pt), flush=True)
