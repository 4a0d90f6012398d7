"""Short Jacobi run for ncu (one GPU): `phases` FUSED phases of the N x N grid, G = 1."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

N = int(os.environ.get("N", 16384))
phases = int(os.environ.get("PHASES", 6))
mech = {v: k for k, v in _lib.MECH_NAMES.items()}[os.environ.get("MECH", "fused")]
torch.cuda.set_device(0)
rt.init(1, 0, rt.new_job_key())
rt.set_config(mech=mech, agent_kernel=int(os.environ.get("AKERN", 1)))
J = wl.Jacobi(N, int(os.environ.get("CHUNK", 128 * 1024)), x0=torch.from_numpy(synth.jacobi_init(N)).cuda(),
              rows_per_tile=int(os.environ.get("RPT", 16)))
s = torch.cuda.Stream()
for k in range(phases):
    J.step(s, barrier=(k == phases - 1))
torch.cuda.synchronize()
rt.check_device()
rt.finalize()
print("prof_jacobi done")
