"""One PageRank configuration per process (loopback G=2): iters, hot, mech from argv; prints
the relative error and a few values per rank.  REPEAT runs it several times in one process."""
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

iters, hot, mech, G = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
src, dst = synth.rmat(12, 16)
V = 1 << 12
want = oracle.pagerank(V, src, dst, iters).astype(np.float64)
for rep in range(int(os.environ.get("REPEAT", 1))):
    def body(r, G_):
        rt.set_config(mech=mech, watchdog_ms=10000)
        s = torch.cuda.Stream()
        P = wl.PageRank(V, src, dst, 4096, stream=s, hot=hot)
        rs = []
        for k in range(iters):
            P.step(s, barrier=(k == iters - 1))
        out = (P.v0, P.v1, P.ranks(s).cpu().numpy())
        rt.check_device()
        P.free()
        return out
    res = []
    for v0, v1, r in run_ranks(G, body, device=0):
        rel = np.abs(r - want[v0:v1]) / want[v0:v1]
        res.append((v0, v1, float(rel.max()), [float(x) for x in r[:2]], [float(x) for x in want[v0:v0 + 2]]))
    print(f"rep={rep} iters={iters} hot={hot} mech={mech} G={G} kernel={os.environ.get('PROACT_PR_KERNEL', 'hot')}: {res}", flush=True)
