#!/usr/bin/env python
"""NEXT-1: overhead / overlap decomposition (Sec. V-C; Sec. IV-B).

For one workload phase at G ranks it measures (median per-phase device time, max over ranks):
  T_local  - the producer alone (no tracking, no transfer)                  [LOCAL]
  T_elide  - tracking + agent, remote stores elided                          [ELIDE]
  T_fused  - PROACT-decoupled (tracking + agent + pushes)                     [FUSED]
  T_inline - PROACT-inline (producer stores to every peer)                    [INLINE]
  T_bulk   - producer, then cudaMemcpy duplication (L245)                     [BULK]
and derives the paper's quantities:
  tracking overhead  = T_elide / T_local - 1                        (Fig. 8)
  infinite-BW bound  = T_bulk - T_copy, T_copy = T_bulk - T_local   (L253)
  transfer overlap   = 1 - (T_fused - T_elide) / T_copy             (Fig. 9)
With all ranks on one GPU (loopback) the "links" are HBM copies; the methodology is the
paper's, the numbers are not NVLink numbers.  One JSON line per workload.

    python tools/decompose.py --workload jacobi|micro [--ranks 2] [--phases 12]
"""
import argparse
import json
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # loopback ranks: see loopback.py
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

MECHS = [("local", _lib.MECH_LOCAL), ("elide", _lib.MECH_ELIDE), ("fused", _lib.MECH_FUSED),
         ("inline", _lib.MECH_INLINE), ("bulk", _lib.MECH_BULK), ("dma", _lib.MECH_DMA)]


def body(r, G, args):
    s = torch.cuda.Stream()
    if args.workload == "jacobi":
        N = args.grid_n
        W = wl.Jacobi(N, args.chunk, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
        step = lambda: W.step(s, barrier=True)  # noqa: E731
    else:
        W = wl.Micro(args.bytes // 4, args.chunk)
        step = lambda: W.step(0x5EED, args.K, False, stream=s, barrier=True)  # noqa: E731
    out = {}
    for name, m in MECHS:
        rt.set_config(mech=m, agent_warps=args.warps)
        ts = []
        for k in range(args.phases):
            rt.host_barrier()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            step()
            b.record(s)
            s.synchronize()
            ts.append(a.elapsed_time(b))
        out[name] = statistics.median(ts[2:])
    rt.check_device()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="jacobi", choices=["jacobi", "micro"])
    ap.add_argument("--ranks", type=int, default=2)
    ap.add_argument("--phases", type=int, default=12)
    ap.add_argument("--grid-n", type=int, default=8192)
    ap.add_argument("--bytes", type=int, default=256 << 20)
    ap.add_argument("--K", type=int, default=1)
    ap.add_argument("--chunk", type=int, default=1 << 20)
    ap.add_argument("--warps", type=int, default=16)
    args = ap.parse_args()
    res = run_ranks(args.ranks, body, args)
    T = {k: max(r[k] for r in res) for k in res[0]}
    t_copy = max(1e-9, T["bulk"] - T["local"])
    line = {"workload": args.workload, "ranks": args.ranks, "loopback": True, "ms": T,
            "tracking_overhead": T["elide"] / T["local"] - 1.0,
            "infinite_bw_ms": T["bulk"] - t_copy, "copy_ms": t_copy,
            "transfer_overlap": 1.0 - (T["fused"] - T["elide"]) / t_copy,
            "speedup_fused_vs_bulk": T["bulk"] / T["fused"], "speedup_fused_vs_inline": T["inline"] / T["fused"],
            "speedup_dma_vs_bulk": T["bulk"] / T["dma"],
            "opportunity_captured": (T["bulk"] - t_copy) / T["fused"]}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
