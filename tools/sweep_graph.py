"""PageRank / SSSP phase-kernel time on RMAT-SCALE for the library variant in $PROACT_LIB."""
import os
import statistics
import sys
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

scale = int(os.environ.get("SCALE", 24))
torch.cuda.set_device(0)
rt.init(1, 0, rt.new_job_key())
src, dst = synth.rmat(scale, 16)
V = 1 << scale
s = torch.cuda.Stream()
P = wl.PageRank(V, src, dst, 131072, stream=s)
ts = []
for k in range(12):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    i = P.k & 1
    a.record(s)
    _lib.check(rt.lib().proact_pagerank_phase(P.gid, P.rid[i], P.rid[i ^ 1], P.d, wl._s(s)), "pr")
    b.record(s)
    rt.phase_sync(s)
    P.k += 1
    ts.append((a, b))
torch.cuda.synchronize()
pr = statistics.median(a.elapsed_time(b) for a, b in ts[2:])
P.free()
w = synth.weights(src.size)
S = wl.SSSP(V, src, dst, w, int(np.bincount(src, minlength=V).argmax()), 131072, stream=s)
t = []
for k in range(6):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    S.step(s)
    b.record(s)
    b.synchronize()
    t.append(a.elapsed_time(b))
print(f"{os.environ.get('PROACT_LIB','default')}: pagerank {pr:.3f} ms  sssp rounds ms {[round(x, 3) for x in t]}", flush=True)
rt.finalize()
