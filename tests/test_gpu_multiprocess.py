"""The multi-PROCESS path: two processes on one GPU map each other's replicas, flags and credits
with CUDA IPC (cudaIpcOpenMemHandle), exactly as one-process-per-GPU torchrun jobs do; the
kernels time-slice on the shared GPU, so this checks correctness, not speed."""
import os
import subprocess
import sys
import uuid

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_two_processes_ipc_jacobi(tmp_path):
    G, N, iters = 2, 256, 4
    job = "mp" + uuid.uuid4().hex[:12]
    procs = []
    for r in range(G):
        env = dict(os.environ, PROACT_RANK=str(r), PROACT_JOB=job, WORLD=str(G), N=str(N),
                   ITERS=str(iters), OUT=str(tmp_path / f"r{r}.npy"), WATCHDOG_MS="90000")
        env.pop("RANK", None)
        procs.append(subprocess.Popen([sys.executable, os.path.join(ROOT, "tools", "mp_rank.py")], env=env,
                                      stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True))
    outs = []
    for p in procs:
        try:
            o, _ = p.communicate(timeout=240)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        outs.append(o)
        assert p.returncode == 0, o
    for o in outs:
        assert "ranks_on_device 2" in o, o
    want = oracle.jacobi(synth.jacobi_init(N), iters)
    for r in range(G):
        got = np.load(tmp_path / f"r{r}.npy")
        assert np.array_equal(got.view(np.uint32), want.view(np.uint32)), r
