import os, sys
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import synth
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl
mode = sys.argv[1]
N, iters = 256, 4
x0 = synth.jacobi_init(N)
def body(r, G):
    rt.set_config(mech=_lib.MECH_FUSED, watchdog_ms=3000)
    s = torch.cuda.Stream()
    if "j" in mode:
        J = wl.Jacobi(N, 4096, x0=torch.from_numpy(x0).cuda())
        if "M" in mode:
            M = wl.Micro(1 << 14, 4096)
        for k in range(iters):
            J.step(s, barrier=(k == iters - 1))
    if "m" in mode or "M" in mode:
        if "m" in mode:
            M = wl.Micro(1 << 14, 4096)
        for _ in range(2):
            M.step(0x5EED, 1, False, stream=s, barrier=True)
    s.synchronize()
    rt.check_device()
ok = 0
for t in range(int(sys.argv[2])):
    try:
        run_ranks(2, body, device=0)
        ok += 1
    except Exception as e:
        print("fail", type(e).__name__, str(e)[:80])
print(mode, "ok", ok)
