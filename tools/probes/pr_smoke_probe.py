"""Relative error of PageRank vs the oracle per rank (loopback G=2) for a few settings."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

src, dst = synth.rmat(12, 16)
V = 1 << 12
for hot in (0, 64, -1):
    for iters in (1, 2, 3, 20):
        for mech in (_lib.MECH_FUSED, _lib.MECH_BULK):
            def body(r, G):
                rt.set_config(mech=mech, watchdog_ms=10000)
                s = torch.cuda.Stream()
                P = wl.PageRank(V, src, dst, 4096, stream=s, hot=hot)
                for k in range(iters):
                    P.step(s, barrier=(k == iters - 1))
                out = (P.v0, P.v1, P.ranks(s).cpu().numpy(), P.nhot)
                rt.check_device()
                P.free()
                return out
            want = oracle.pagerank(V, src, dst, iters).astype(np.float64)
            res = []
            for v0, v1, r, nh in run_ranks(2, body, device=0):
                rel = np.abs(r - want[v0:v1]) / want[v0:v1]
                res.append((v0, v1, nh, float(rel.max()), int((rel > 1e-5).sum())))
            print(f"hot={hot} iters={iters} mech={mech}: {res}", flush=True)
