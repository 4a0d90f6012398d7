"""Agent vs producer timeline per Jacobi phase (G = 1, ELIDE), from a -DPROACT_TIMING_EXP build
(PROACT_LIB=.../libproact_texp.so, PROACT_DEBUG=2): agent first start / last exit, producer CTA
first start / last exit / mean CTA duration, per agent placement and agent warps."""
import ctypes
import os
import sys
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

N = 16384
torch.cuda.set_device(0)
rt.init(1, 0, rt.new_job_key())
J = wl.Jacobi(N, 131072, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
s = torch.cuda.Stream()
arr = (ctypes.c_ulonglong * 8)()
M = (1 << 64) - 1
for ak in (0, 1):
    for w in (4, 16, 64):
        rt.set_config(mech=_lib.MECH_ELIDE, agent_warps=w, agent_kernel=ak)
        for _ in range(3):
            J.step(s)
        s.synchronize()
        rows = []
        for _ in range(5):
            rt.lib().proact_debug_agent_prof(arr)
            J.step(s)
            s.synchronize()
            rt.lib().proact_debug_agent_prof(arr)
            a = list(arr)
            a0, a1, p0, p1 = M - a[0], a[1], M - a[2], a[3]
            t0 = min(a0, p0)
            rows.append((a0 - t0, a1 - t0, p0 - t0, p1 - t0, a[4] / max(1, a[5]), a[5]))
        r = rows[-1]
        print(f"akern={ak} warps={w}: agent [{r[0] / 1e3:.1f}, {r[1] / 1e3:.1f}] us, producer [{r[2] / 1e3:.1f}, "
              f"{r[3] / 1e3:.1f}] us, mean CTA {r[4] / 1e3:.1f} us over {r[5]} CTAs", flush=True)
rt.check_device()
rt.finalize()
