"""Runtime pieces beyond the kernels: the profiler (a9) and bench.py's multi-process path."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch

import oracle
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_autotune_sweeps_caches_and_keeps_results_correct(tmp_path, monkeypatch):
    """proact_autotune (Sec. III-A): brute force over mechanism x chunk x
    agent warps, max-over-ranks time, JSON cache keyed by workload; results stay bit-exact for
    every point (the callback checks them)."""
    cache = tmp_path / "tune.json"
    monkeypatch.setenv("PROACT_TUNE_CACHE", str(cache))
    W = 1 << 20
    seen = []

    def body(r, G):
        M = wl.Micro(W, 65536)
        s = torch.cuda.Stream()

        def run(cfg):
            if cfg["chunk_bytes"] != rt.region_info(M.rid).chunk_bytes:
                rt.rechunk(M.rid, cfg["chunk_bytes"])
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            for _ in range(3):
                M.step(0x5EED, 1, False, stream=s, barrier=True)
            b.record(s)
            s.synchronize()
            rt.host_barrier()
            want = oracle.micro_phase(W, M.phase - 1, 0x5EED, 1)
            assert np.array_equal(M.buf.cpu().numpy().view(np.uint32), want)
            rt.host_barrier()
            if r == 0:
                seen.append(dict(cfg))
            return a.elapsed_time(b)

        best = rt.autotune("micro_1M_G2", run, "mech=0,1;warps=4,16;chunk=65536,262144")
        again = rt.autotune("micro_1M_G2", run, None)   # cached: no new runs
        return best, again

    n_before = len(seen)
    outs = run_ranks(2, body)
    (best0, again0), (best1, _) = outs
    assert best0 == best1 and again0["mech"] == best0["mech"]
    assert best0["mech"] in (_lib.MECH_FUSED, _lib.MECH_INLINE)
    assert best0["chunk_bytes"] in (65536, 262144)
    # FUSED: 2 chunks x 2 warps points; INLINE: 2 chunks (warps ignored) -> 6 runs, cache hit after
    assert len(seen) - n_before == 6
    d = json.loads(cache.read_text())
    assert "micro_1M_G2" in d and d["micro_1M_G2"]["chunk_bytes"] == best0["chunk_bytes"]


@pytest.mark.slow
def test_bench_two_processes_json_line():
    """bench.py --gpus 2 under torchrun (both ranks on this one GPU: CUDA IPC, time-sliced)."""
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    env = dict(os.environ, PROACT_BENCH_SAME_DEVICE="1", PROACT_WATCHDOG_MS="120000")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "1", "--warmup", "3", "--grid-n", "1024", "--iters", "4", "--backend", "gloo",
           "--no-cpu"]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["scaling"] == "strong"
    # e2e through both host-buffer entry points (sequential and pipelined), two processes
    assert d["e2e"]["value"] > 0 and d["e2e"]["sequential_value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 513 * 1024 * 4   # rank 0: its rows + one halo row
    # the same ranks time the bulk-copy and naive-P2P baselines (NCCL needs distinct GPUs)
    assert set(d["baselines_iters_per_s"]) == {"bulk_cudaMemcpyPeer", "naive_p2p_inline"}
    assert all(v > 0 for v in d["baselines_iters_per_s"].values())
    # strong scaling against the single-GPU solve measured in the same run
    assert d["speedup_vs_n1"] > 0 and d["n1_reference"]["value"] > 0
    sr = d["step_roofline"]
    assert 0 < sr["frac"] and sr["nvlink_ingress_GBps_per_gpu"] > 0 and sr["t_nvl_us"] > 0
    # the profiler swept push engine x agent placement (incl. the producer-CTA transfer warps)
    assert "push=0,1" in d["config"]["tuned"]["space"] and "akern=0,1,2" in d["config"]["tuned"]["space"]
    # halo-only variant beside full replication, with its own baselines and roofline
    h = d["halo_only"]
    assert h["value"] > 0 and h["speedup_vs_n1"] > 0 and h["step_roofline"]["frac"] > 0
    assert "warps=1,2,4" in h["tuned"]["space"] and h["tuned"]["best"]["agent_kernel"] in (0, 1, 2)
    assert set(h["baselines_iters_per_s"]) == {"bulk_cudaMemcpyPeer", "naive_p2p_inline"}
    assert d["agent_cost"]["agent_sm_ms_per_GB_pushed"] >= 0
    dc = d["decomposition"]   # NEXT-1: infinite-bandwidth bound, tracking overhead, captured
    assert dc["ms_per_phase"]["local_no_transfer"] > 0 and dc["ms_per_phase"]["elide_tracking_only"] > 0
    assert "opportunity_captured" in dc
