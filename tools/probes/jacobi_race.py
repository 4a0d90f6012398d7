"""Repeat a small G = 2 loopback Jacobi solve (N = 512, 7 phases, 16 KiB chunks) and count results
that differ from the oracle: MODE=class (replicas preloaded, Jacobi class) or MODE=host
(proact_jacobi_solve_host); PROACT_* env selects the mechanism."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

N, iters, chunk = int(os.environ.get("N", 512)), 7, int(os.environ.get("CHUNK", 16384))
mode = os.environ.get("MODE", "class")
x0 = synth.jacobi_init(N)
want = oracle.jacobi(x0, iters)


def body(r, G):
    s = torch.cuda.Stream()
    if mode == "host":
        xh = torch.from_numpy(x0).pin_memory()
        out = torch.zeros((N, N), dtype=torch.float32).pin_memory()
        wl.jacobi_solve_host(xh, out, N, iters, chunk, stream=s)
        s.synchronize()
        r0, r1 = wl.row_split(N, G, r)
        return out.numpy()[r0:r1].copy(), r0, r1
    J = wl.Jacobi(N, chunk, x0=torch.from_numpy(x0).cuda())
    rt.host_barrier()
    for k in range(iters):
        J.step(s, barrier=(k == iters - 1))
    s.synchronize()
    r0, r1 = J.r0, J.r1
    return J.current.cpu().numpy()[r0:r1].copy(), r0, r1


bad = 0
reps = int(os.environ.get("REPS", 40))
for k in range(reps):
    for rows, r0, r1 in run_ranks(2, body):
        if not np.array_equal(rows, want[r0:r1]):
            diff = np.nonzero((rows != want[r0:r1]).any(1))[0] + r0
            print("mismatch rank rows", r0, r1, "bad rows", diff[:10].tolist(), flush=True)
            bad += 1
print(f"MODE={mode} N={N} chunk={chunk} bad={bad}/{reps}", flush=True)
