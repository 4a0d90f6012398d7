"""Host issue cost vs device time per Jacobi phase (G = 1), per mechanism: is a step launch-bound?"""
import os
import sys
import time
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # before torch: see bench.py

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

N = int(os.environ.get("N", 16384))
I = 100
torch.cuda.set_device(0)
rt.init(1, 0, rt.new_job_key())
J = wl.Jacobi(N, 131072, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
s = torch.cuda.Stream()
for mech in os.environ.get("MECHS", "local,elide,fused,elide0").split(","):
    ak = 0 if mech.endswith("0") else 1
    mech = mech.rstrip("0")
    rt.set_config(mech={v: k for k, v in _lib.MECH_NAMES.items()}[mech], agent_kernel=ak)
    for _ in range(2):
        for k in range(I):
            J.step(s, barrier=(k == I - 1))
    torch.cuda.synchronize()
    # host issue cost: enqueue behind a long sleep so the device never throttles the host
    t0 = time.perf_counter()
    for k in range(I):
        J.step(s, barrier=(k == I - 1))
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for k in range(I):
        J.step(s, barrier=(k == I - 1))
    b.record(s)
    torch.cuda.synchronize()
    # device time of the kernels alone (events around each jacobi_phase)
    evs = []
    for k in range(I):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        i = J.k & 1
        e0.record(s)
        wl.jacobi_phase(J.rid[i], J.rid[i ^ 1], N, 16, s)
        e1.record(s)
        rt.phase_sync(s, barrier=(k == I - 1))
        J.k += 1
        evs.append((e0, e1))
    torch.cuda.synchronize()
    kern = sum(x.elapsed_time(y) for x, y in evs) / I
    tot = evs[0][0].elapsed_time(evs[-1][1]) / (I - 1) * 1000
    gaps = sorted(evs[k][1].elapsed_time(evs[k + 1][0]) * 1000 for k in range(I - 1))
    print(f"  {mech}: kernel-loop {tot:.1f} us/phase, gap e1->next e0 median {gaps[len(gaps)//2]:.1f} max {gaps[-1]:.1f} us")
    print(f"{mech}: host issue {1e6 * (t1 - t0) / I:.1f} us/phase, step {a.elapsed_time(b) / I * 1000:.1f} us/phase, "
          f"kernel {kern * 1000:.1f} us/phase", flush=True)
rt.check_device()
rt.finalize()
