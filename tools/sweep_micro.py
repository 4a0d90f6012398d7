"""Loopback transfer microbenchmark sweep (config 5 shape on one GPU): G ranks as threads,
each produces R/G bytes per phase and the agents replicate them to the other G-1 ranks
(HBM -> HBM here; no NVLink on a one-GPU box).  Prints one JSON line per point:
replicated GB/s = (G-1) * R / phase time, per mechanism / chunk / agent warps / discovery."""
import itertools
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # loopback ranks: see loopback.py
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

G = int(os.environ.get("G", 2))
R = int(os.environ.get("RBYTES", 256 << 20))
K = int(os.environ.get("K", 1))
chunks = [int(x) for x in os.environ.get("CHUNKS", "65536,1048576").split(",")]
mechs = os.environ.get("MECHS", "fused,inline,bulk,elide").split(",")
warps = [int(x) for x in os.environ.get("WARPS", "8,32").split(",")]
discs = [int(x) for x in os.environ.get("DISCS", "0").split(",")]
pieces = [int(x) for x in os.environ.get("PIECES", "65536").split(",")]
pushes = [int(x) for x in os.environ.get("PUSHES", "0").split(",")]
akerns = [int(x) for x in os.environ.get("AKERNS", "0").split(",")]
PH = int(os.environ.get("PHASES", 6))


def body(r, G_):
    M = wl.Micro(R // 4, chunks[0])
    s = torch.cuda.Stream()
    out = []
    for ch in chunks:
        if ch != rt.region_info(M.rid).chunk_bytes:
            rt.rechunk(M.rid, ch)
        for mech, w, d, pc, pu, ak in itertools.product(mechs, warps, discs, pieces, pushes, akerns):
            agent = mech in ("fused", "elide")
            if not agent and (w != warps[0] or d != discs[0] or pc != pieces[0] or pu != pushes[0] or ak != akerns[0]):
                continue
            rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[mech], agent_warps=w, discovery=d,
                          piece_bytes=pc, push=pu, agent_kernel=ak)
            ts = []
            if os.environ.get("PROACT_DEBUG") == "2":
                import ctypes
                rt.lib().proact_debug_agent_prof((ctypes.c_ulonglong * 8)())
            for k in range(PH):
                rt.host_barrier()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                M.step(0x5EED, K, False, stream=s, barrier=True)
                b.record(s)
                s.synchronize()
                ts.append(a.elapsed_time(b))
            prof = None
            if os.environ.get("PROACT_DEBUG") == "2":
                import ctypes
                arr = (ctypes.c_ulonglong * 8)()
                rt.lib().proact_debug_agent_prof(arr)
                prof = list(arr)[:6]
            out.append({"prof": prof, "chunk": ch, "mech": mech, "warps": w, "disc": d, "piece": pc, "push": pu, "akern": ak,
                        "ms": statistics.median(ts[2:])})
    return out


res = run_ranks(G, body)
for i, pt in enumerate(res[0]):
    ms = max(res[g][i]["ms"] for g in range(G))
    pt.update({"G": G, "R": R, "K": K, "ms": ms, "GBps_repl": (G - 1) * R / ms / 1e6})
    print(json.dumps(pt), flush=True)
