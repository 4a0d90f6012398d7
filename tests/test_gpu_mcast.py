"""NVLS multicast pushes: replicas from proact_alloc_replica bound to one
multicast object; the agent's multimem.st.global.v4 stores reach every peer through the NVSwitch.
Needs >= 2 GPUs of a multicast-capable (NVSwitch) system: skipped elsewhere.  The fallback path
(proact_alloc_replica without multicast, PUSH_MULTICAST degrading to unicast stores) runs on any
box, loopback included."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl

pytestmark = pytest.mark.gpu
SEED = 0x5EED


def _body(r, G, words, chunk, phases):
    rt.set_config(mech=_lib.MECH_FUSED, push=_lib.PUSH_MULTICAST, agent_kernel=_lib.AGENT_SEPARATE, agent_warps=8)
    supported = rt.mcast_supported()
    buf = rt.alloc_replica((words,), torch.int32)
    buf.zero_()
    torch.cuda.synchronize()
    bounds = [((words * p) // G) // 4 * 4 for p in range(G)] + [words]
    rid = rt.register_region(buf, bounds[r] * 4, (bounds[r + 1] - bounds[r]) * 4, chunk)
    s = torch.cuda.Stream()
    snaps = []
    for p in range(phases):
        wl.micro_phase(rid, p, SEED, 1, False, s)
        rt.phase_sync(s, barrier=True)
        s.synchronize()
        snaps.append(buf.cpu().numpy().view(np.uint32).copy())
        rt.host_barrier()
    rt.check_device()
    rt.free_replica(buf)
    return supported, snaps


def _check(outs, words, phases):
    for p in range(phases):
        want = oracle.micro_phase(words, p, SEED, 1)
        for g, (_, snaps) in enumerate(outs):
            assert np.array_equal(snaps[p], want), (p, g)


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="NVLS multicast needs >= 2 GPUs on an NVSwitch")
def test_multicast_push_replicates_to_every_gpu():
    G = min(torch.cuda.device_count(), 8)
    words = 1 << 22
    outs = run_ranks(G, _body, words, 1 << 20, 3, device=list(range(G)))
    if not all(sup for sup, _ in outs):
        pytest.skip("devices do not report CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED")
    _check(outs, words, 3)


def test_multicast_push_falls_back_to_unicast_in_loopback():
    """Loopback ranks share one device (no switch): proact_alloc_replica returns plain replicas,
    PUSH_MULTICAST pushes with 16-byte unicast stores -- the bytes are still right."""
    words = (1 << 20) + 4 * 3
    outs = run_ranks(2, _body, words, 65536, 3)
    assert not any(sup for sup, _ in outs)
    _check(outs, words, 3)
