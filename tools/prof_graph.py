"""Short PageRank / SSSP run for ncu (one GPU): WORKLOAD=pagerank|sssp, SCALE, PHASES."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

scale = int(os.environ.get("SCALE", 24))
phases = int(os.environ.get("PHASES", 4))
chunk = int(os.environ.get("CHUNK", 128 * 1024))
torch.cuda.set_device(0)
rt.init(1, 0, rt.new_job_key())
src, dst = synth.rmat(scale, 16)
V = 1 << scale
s = torch.cuda.Stream()
if os.environ.get("WORKLOAD", "pagerank") == "pagerank":
    P = wl.PageRank(V, src, dst, chunk, stream=s)
    for k in range(phases):
        P.step(s, barrier=(k == phases - 1))
else:
    w = synth.weights(src.size)
    S = wl.SSSP(V, src, dst, w, int(np.bincount(src, minlength=V).argmax()), chunk, stream=s)
    for k in range(phases):
        S.step(s)
torch.cuda.synchronize()
rt.check_device()
rt.finalize()
print("prof_graph done")
