"""GPU parity for the banded-matrix Jacobi (NEXT-2) vs the oracle, bit-exact
(reading R19: fixed order, no FMA, IEEE division)."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl

pytestmark = pytest.mark.gpu


def _body(r, G, N, w, iters, chunk, mech):
    rt.set_config(mech=mech)
    a, b = synth.banded(N, w)
    B = wl.Banded(a, b, chunk)
    s = torch.cuda.Stream()
    for k in range(iters):
        B.step(s, barrier=(k == iters - 1))
    s.synchronize()
    rt.check_device()
    return B.current.cpu().numpy(), (B.r0, B.r1)


@pytest.mark.parametrize("G,N,w,chunk,mech", [(1, 5000, 3, 4096, _lib.MECH_FUSED), (2, 20000, 16, 4096, _lib.MECH_FUSED),
                                              (3, 9999 // 4 * 4, 64, 8192, _lib.MECH_FUSED),
                                              (4, 12000, 700, 4096, _lib.MECH_FUSED),   # band wider than a slice
                                              (2, 8000, 8, 4096, _lib.MECH_INLINE), (2, 8000, 8, 4096, _lib.MECH_BULK),
                                              (1, 4096, 0, 4096, _lib.MECH_FUSED),      # no off-diagonals
                                              (2, 20000, 4200, 4096, _lib.MECH_FUSED)])  # w > 4096: banded_kernel
def test_banded_jacobi_bit_exact(G, N, w, chunk, mech):
    iters = 7
    a, b = synth.banded(N, w)
    want = oracle.banded_jacobi(a, b, np.zeros(N, np.float32), iters)
    outs = run_ranks(G, _body, N, w, iters, chunk, mech)
    for g, (x, _) in enumerate(outs):
        assert np.array_equal(x.view(np.uint32), want.view(np.uint32)), g


def test_banded_tma_and_plain_kernels_agree(monkeypatch):
    """banded_tma_kernel (default) and banded_kernel (PROACT_BANDED_PLAIN=1, read once per
    process, so each runs in its own subprocess) give bit-identical iterates."""
    import os
    import subprocess
    import sys
    code = ("import sys, numpy as np, torch; sys.path.insert(0, %r);"
            "import synth; from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt, workloads as wl;"
            "torch.cuda.set_device(0); rt.init(1, 0, rt.new_job_key()); a, b = synth.banded(65536, 24);"
            "B = wl.Banded(a, b, 131072); s = torch.cuda.Stream();"
            "[B.step(s, barrier=(k == 4)) for k in range(5)]; s.synchronize();"
            "sys.stdout.buffer.write(B.current.cpu().numpy().tobytes()); rt.finalize()"
            % os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    outs = []
    for plain in ("0", "1"):
        env = dict(os.environ, PROACT_BANDED_PLAIN=plain)
        outs.append(subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, timeout=300,
                                   check=True).stdout)
    assert len(outs[0]) == 65536 * 4 and outs[0] == outs[1]
