"""One rank of tests/test_gpu_jacobi.py::test_jacobi_allgather_baseline (launched by torchrun):
the NCCL all-gather Jacobi baseline on GPU `LOCAL_RANK`, compared with the oracle."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

rank, world, local = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"]), int(os.environ["LOCAL_RANK"])
torch.cuda.set_device(local)
dist.init_process_group("nccl", device_id=torch.device("cuda", local))
rt.init(world, rank, f"allgather_{os.environ['MASTER_PORT']}")
rt.set_config(mech=_lib.MECH_LOCAL)
N, iters = 1024, 10
J = wl.Jacobi(N, 65536, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
s = torch.cuda.Stream()
for _ in range(iters):
    J.step_allgather(s)
s.synchronize()
got = J.current.cpu().numpy()
want = oracle.jacobi(synth.jacobi_init(N), iters)
assert np.array_equal(got.view(np.uint32), want.view(np.uint32)), "all-gather replica != oracle"
rt.finalize()
dist.destroy_process_group()
print("ALLGATHER_OK", flush=True)
