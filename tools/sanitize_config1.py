"""Config 1 (Jacobi 1024^2, G = 2 loopback ranks, 10 iterations) for compute-sanitizer: every
mechanism / agent placement once, results checked against the oracle.  G = 1 with PROACT_G1=1.

    compute-sanitizer --tool memcheck python tools/sanitize_config1.py
"""
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

G = 1 if os.environ.get("PROACT_G1") == "1" else 2
N, iters = 1024, 10
CFGS = [dict(mech=_lib.MECH_FUSED, agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_BULK),
        dict(mech=_lib.MECH_FUSED, agent_kernel=_lib.AGENT_SEPARATE, push=_lib.PUSH_VEC16),
        dict(mech=_lib.MECH_FUSED, agent_kernel=_lib.AGENT_PRODUCER),
        dict(mech=_lib.MECH_INLINE), dict(mech=_lib.MECH_BULK), dict(mech=_lib.MECH_DMA)]
if G == 1:
    CFGS = [dict(mech=_lib.MECH_ELIDE, agent_kernel=a) for a in (0, 1, 2)] + [dict(mech=_lib.MECH_LOCAL)]
want = oracle.jacobi(synth.jacobi_init(N), iters)


def body(r, G_):
    out = []
    for cfg in CFGS:
        rt.set_config(watchdog_ms=60000, **cfg)
        J = wl.Jacobi(N, 65536, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
        s = torch.cuda.Stream()
        for k in range(iters):
            J.step(s, barrier=(k == iters - 1))
        s.synchronize()
        rt.check_device()
        out.append(np.array_equal(J.current.cpu().numpy().view(np.uint32), want.view(np.uint32)))
        rt.host_barrier()
        if len(out) * 2 + 2 > _lib.MAX_REGIONS:   # regions cannot be unregistered: one config per context
            break
    return out


res = []
for k in range(0, len(CFGS), 3):
    sub = CFGS[k:k + 3]
    CFGS_ALL, CFGS = CFGS, sub
    res += [x for per in zip(*run_ranks(G, body, timeout=1200)) for x in [all(per)]]
    CFGS = CFGS_ALL
print("sanitize_config1: G =", G, "results vs oracle:", res, flush=True)
assert all(res)
