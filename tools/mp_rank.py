"""One rank of a multi-PROCESS PROACT job (CUDA IPC path), used by tests/test_gpu_multiprocess.py.

env: PROACT_RANK, PROACT_JOB, WORLD, N, ITERS, OUT (path of the .npy result), DEVICE.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

torch.cuda.set_device(int(os.environ.get("DEVICE", "0")))
G, N, iters = int(os.environ["WORLD"]), int(os.environ["N"]), int(os.environ["ITERS"])
rt.init(G)   # rank and job from $PROACT_RANK / $PROACT_JOB
rt.set_config(watchdog_ms=int(os.environ.get("WATCHDOG_MS", "60000")))
J = wl.Jacobi(N, 4096, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
s = torch.cuda.Stream()
for k in range(iters):
    J.step(s, barrier=(k == iters - 1))
s.synchronize()
rt.check_device()
np.save(os.environ["OUT"], J.current.cpu().numpy())
print("rank", rt.rank(), "ranks_on_device", rt.ranks_on_device(), "ok", flush=True)
rt.finalize()
