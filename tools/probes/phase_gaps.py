"""Per-phase timeline of the bench step (config 2, G = 1): CUDA events before / after every
jacobi_phase launch and after every phase_sync on the launching stream -> kernel time and the
gap between consecutive kernels.  PROACT_SYNC_KERNEL=1 swaps the single-rank memory-op sync for
the 1-warp sync kernel."""
import os
import statistics
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

N = int(os.environ.get("N", 16384))
torch.cuda.set_device(0)
rt.init(1, 0, rt.new_job_key())
rt.set_config(mech=_lib.MECH_FUSED, chunk_bytes=131072)
J = wl.Jacobi(N, 131072, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
s = torch.cuda.Stream()
for _ in range(20):
    J.step(s)
torch.cuda.synchronize()
P = 100
ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(P)]
for k in range(P):
    i = J.k & 1
    ev[k][0].record(s)
    wl.jacobi_phase(J.rid[i], J.rid[i ^ 1], N, J.rpt, s)
    ev[k][1].record(s)
    rt.phase_sync(s)
    ev[k][2].record(s)
    J.k += 1
torch.cuda.synchronize()
kern = [ev[k][0].elapsed_time(ev[k][1]) * 1e3 for k in range(P)]
sync = [ev[k][1].elapsed_time(ev[k][2]) * 1e3 for k in range(P)]
gap = [ev[k][2].elapsed_time(ev[k + 1][0]) * 1e3 for k in range(P - 1)]
tot = ev[0][0].elapsed_time(ev[P - 1][2]) * 1e3 / P
print(f"sync_kernel={os.environ.get('PROACT_SYNC_KERNEL', '0')} per phase {tot:.1f} us: kernel median "
      f"{statistics.median(kern):.1f} us, sync {statistics.median(sync):.1f} us, gap {statistics.median(gap):.1f} us")
rt.finalize()
