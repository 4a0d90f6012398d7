"""World-size-2 CPU tests (gloo) of the N > 1 host logic: the /dev/shm rendezvous that
proact_init uses, the region slice plan, the graph destination partition, and bench.py's
max-over-ranks timing -- each rank computes independently and the results are cross-checked
through torch.distributed (gloo).  No GPU is needed (host-only library entry points)."""
import ctypes
import os
import socket
import uuid

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_isca_muthukrishnannl21_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, job, q):
    try:
        import sys
        sys.path.insert(0, ROOT)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        L = _lib.load()
        # 1. the shm rendezvous agrees with gloo's all_gather
        mine = np.array([rank * 1000 + 7, rank ** 2 + 1], dtype=np.uint64)
        allv = np.zeros((world, 2), dtype=np.uint64)
        rc = L.proact_rdv_allgather(job.encode(), world, rank, mine.ctypes.data, mine.nbytes, allv.ctypes.data)
        assert rc == 0, rc
        ref = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(ref, torch.from_numpy(mine.astype(np.int64)))
        assert np.array_equal(allv.astype(np.int64), torch.stack(ref).numpy())
        # 2. slice plan: every rank derives the same offsets / chunk numbering from the gathered bytes
        words = 3_000_000 + 4 * 7
        bounds = [((words * p) // world) // 4 * 4 for p in range(world)] + [words]
        my_bytes = (bounds[rank + 1] - bounds[rank]) * 4
        got = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(got, torch.tensor([my_bytes], dtype=torch.int64))
        b = (ctypes.c_uint64 * world)(*[int(x.item()) for x in got])
        off = (ctypes.c_uint64 * (world + 1))()
        c0 = (ctypes.c_uint32 * (world + 1))()
        chunk = 65536
        assert L.proact_plan_slices(world, b, chunk, off, c0) == 0
        assert off[rank] == bounds[rank] * 4 and off[world] == words * 4
        for p in range(world):
            assert c0[p + 1] - c0[p] == -(-b[p] // chunk)
        plans = [None] * world
        dist.all_gather_object(plans, (list(off), list(c0)))
        assert all(pl == plans[0] for pl in plans)
        # 3. graph partition bounds identical on every rank and in-edge balanced
        import synth
        _, dst = synth.rmat(12, 16)
        V = 1 << 12
        indeg = np.bincount(dst, minlength=V).astype(np.uint32)
        bd = (ctypes.c_uint * (world + 1))()
        assert L.proact_partition_bounds(indeg.ctypes.data, V, world, 256, bd) == 0
        bl = list(bd)
        assert bl[0] == 0 and bl[-1] == V and all(x % 256 == 0 or x == V for x in bl)
        allb = [None] * world
        dist.all_gather_object(allb, bl)
        assert all(x == allb[0] for x in allb)
        share = [int(indeg[bl[p]:bl[p + 1]].sum()) for p in range(world)]
        assert max(share) <= dst.size / world + int(indeg.max()) + 256 * 64
        # 4. bench.py's whole-job time is the max over ranks
        import bench
        assert bench.max_over_ranks(10.0 + rank, world) == 10.0 + world - 1
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # surfaced by the parent
        import traceback
        q.put((rank, traceback.format_exc()))


def test_world2_gloo_host_logic():
    world, port, job = 2, _free_port(), "gloo" + uuid.uuid4().hex[:12]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, job, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in ps:
        p.join(60)
    for r in range(world):
        assert res[r] == "ok", res[r]


def test_partition_bounds_edge_cases():
    L = _lib.load()
    # all edges into one vertex: every split lands on an aligned boundary, monotone
    V = 1024
    indeg = np.zeros(V, dtype=np.uint32)
    indeg[700] = 100
    bd = (ctypes.c_uint * 5)()
    assert L.proact_partition_bounds(indeg.ctypes.data, V, 4, 64, bd) == 0
    b = list(bd)
    assert b[0] == 0 and b[-1] == V and b == sorted(b)
    # G = 1 and empty graph
    bd1 = (ctypes.c_uint * 2)()
    assert L.proact_partition_bounds(np.zeros(V, np.uint32).ctypes.data, V, 1, 64, bd1) == 0
    assert list(bd1) == [0, V]
