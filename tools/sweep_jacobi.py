"""Per-launch jacobi_kernel time (CUDA events) across mechanism / agent warps / tile rows, G = 1."""
import itertools
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # loopback ranks: see loopback.py
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

N = int(os.environ.get("N", 16384))
torch.cuda.set_device(0)
rt.init(1, 0, rt.new_job_key())
chunks = [int(x) for x in os.environ.get("CHUNKS", "131072").split(",")]
J = wl.Jacobi(N, chunks[0], x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
s = torch.cuda.Stream()
mechs = os.environ.get("MECHS", "local,fused,elide").split(",")
warps = [int(x) for x in os.environ.get("WARPS", "1,4,16").split(",")]
rpts = [int(x) for x in os.environ.get("RPTS", "16,64").split(",")]
discs = [int(x) for x in os.environ.get("DISCS", "0").split(",")]
akerns = [int(x) for x in os.environ.get("AKERNS", "1").split(",")]   # 0 FUSED, 1 SEPARATE
res = []
for ch in chunks:
    if ch != rt.region_info(J.rid[0]).chunk_bytes:
        rt.rechunk(J.rid[0], ch)
        rt.rechunk(J.rid[1], ch)
    for mech, w, rpt, disc, ak in itertools.product(mechs, warps, rpts, discs, akerns):
        if mech == "local" and (w != warps[0] or disc != discs[0] or ak != akerns[0]):
            continue
        rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[mech], agent_warps=w, discovery=disc,
                      agent_kernel=ak)
        J.rpt = rpt
        evs = []
        for k in range(24):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            i = J.k & 1
            a.record(s)
            wl.jacobi_phase(J.rid[i], J.rid[i ^ 1], N, rpt, s)
            b.record(s)
            rt.phase_sync(s)
            J.k += 1
            evs.append((a, b))
        torch.cuda.synchronize()
        t = [a.elapsed_time(b) for a, b in evs[4:]]
        ms = statistics.median(t)
        r = {"chunk": ch, "mech": mech, "warps": w, "rpt": rpt, "disc": disc, "akern": ak, "ms": ms, "GBps": 8.0 * N * N / ms / 1e6}
        res.append(r)
        print(json.dumps(r), flush=True)
rt.check_device()
rt.finalize()
