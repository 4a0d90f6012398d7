"""Run G PROACT ranks as threads of one process (one rank per thread).

With all ranks on one GPU ("loopback") the peers' replicas are other buffers of
the same device: every kernel, flag, credit and agent push of the multi-GPU
protocol runs unchanged, only the bytes cross HBM instead of NVLink.  The
library splits the device between the co-resident ranks (grid capacity / G) so
that cross-rank spins always make progress.  This is how the whole protocol is
exercised on the single-GPU boxes this project is tested on.
"""
from __future__ import annotations

import os
import threading

# Several ranks in one process share the device's hardware work queues; with the default 8
# connections, streams of different ranks alias onto one queue and a rank's stream waiting on
# a cross-rank flag can block another rank's queued launch (a false dependency -> deadlock).
# 32 connections (the maximum) must be requested before the CUDA context is created.
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

import torch

from . import runtime as rt


def run_ranks(G: int, fn, *args, device: int = 0, job: str | None = None, timeout: float = 600.0,
              **kw):
    """Call fn(rank, G, *args, **kw) on G threads, each an initialised PROACT rank on
    `device` (an int, or a list of G ints).  Returns the list of results; re-raises the first
    exception."""
    job = job or rt.new_job_key()
    devs = device if isinstance(device, (list, tuple)) else [device] * G
    results = [None] * G
    errors: list[BaseException | None] = [None] * G

    def body(r: int):
        try:
            torch.cuda.set_device(devs[r])
            rt.init(G, r, job)
            try:
                results[r] = fn(r, G, *args, **kw)
            finally:
                torch.cuda.synchronize()
                rt.finalize()
        except BaseException as e:  # noqa: BLE001 - surfaced below
            errors[r] = e

    th = [threading.Thread(target=body, args=(r,), daemon=True) for r in range(G)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout)
    if any(t.is_alive() for t in th):
        raise TimeoutError(f"loopback ranks did not finish within {timeout}s")
    bad = [(r, e) for r, e in enumerate(errors) if e is not None]
    if bad:
        if len(bad) > 1:   # a rank's failure often makes the others time out: report them all
            import sys
            for r, e in bad[1:]:
                print(f"[loopback] rank {r} also failed: {type(e).__name__}: {e}", file=sys.stderr)
        r0, e0 = min(bad, key=lambda x: 0 if not isinstance(x[1], Exception) or "TIMEOUT" not in str(x[1]) else 1)
        raise e0
    return results
