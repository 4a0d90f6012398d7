#!/usr/bin/env python
"""E8 analogue (Table II): run the brute-force profiler (proact_autotune) per
workload at G loopback ranks on this GPU and print a Markdown table of the chosen configuration.

    python tools/tune_table.py [--ranks 2] [--out profiles/r01_tune_table.md]

Loopback: the ranks share one GPU, so "transfers" are HBM copies -- the table documents the
profiler at work on this box, not NVLink optima.
"""
import argparse
import os
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # loopback ranks: see loopback.py
import sys
import tempfile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import _lib, run_ranks  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt  # noqa: E402
from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl  # noqa: E402

SPACE = "mech=0,1,2,5;chunk=131072,1048576,16777216;warps=8,32;piece=65536;push=0,1;disc=0;akern=0,1,2"
NAMES = {v: k for k, v in _lib.MECH_NAMES.items()}


def timed(s, fn, reps=4):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    rt.host_barrier()
    a.record(s)
    for _ in range(reps):
        fn()
    b.record(s)
    s.synchronize()
    rt.host_barrier()
    return a.elapsed_time(b) / reps


def body(r, G, work):
    s = torch.cuda.Stream()
    if work == "jacobi":
        N = 8192
        W = wl.Jacobi(N, 1 << 20, x0=torch.from_numpy(synth.jacobi_init(N)).cuda())
        rids = W.rid
        step = lambda: W.step(s, barrier=True)  # noqa: E731
    elif work == "micro":
        W = wl.Micro((256 << 20) // 4, 1 << 20)
        rids = [W.rid]
        step = lambda: W.step(0x5EED, 1, False, stream=s, barrier=True)  # noqa: E731
    else:
        src, dst = synth.rmat(20, 16)
        W = wl.PageRank(1 << 20, src, dst, 1 << 20, stream=s)
        rids = W.rid
        step = lambda: W.step(s, barrier=True)  # noqa: E731

    def run(cfg):
        for rid in rids:
            if cfg["chunk_bytes"] != rt.region_info(rid).chunk_bytes:
                rt.rechunk(rid, cfg["chunk_bytes"])
        return timed(s, step)

    best = rt.autotune(f"{work}_G{G}_loopback", run, SPACE)
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, default=2)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    os.environ["PROACT_TUNE_CACHE"] = os.path.join(tempfile.mkdtemp(), "tune.json")
    rows = []
    for work in ("micro", "jacobi", "pagerank"):
        best = run_ranks(args.ranks, body, work)[0]
        rows.append((work, best))
    import json
    cache = json.load(open(os.environ["PROACT_TUNE_CACHE"]))
    lines = ["| workload (G loopback) | mechanism | placement | push | chunk | agent warps | phase ms |",
             "|---|---|---|---|---|---|---|"]
    place = {0: "agent CTAs in the grid", 1: "separate agent kernel", 2: "producer-CTA transfer warps"}
    for work, b in rows:
        ms = cache.get(f"{work}_G{args.ranks}_loopback", {}).get("ms")
        agent = b["mech"] in (_lib.MECH_FUSED, _lib.MECH_ELIDE)
        lines.append(f"| {work} (G={args.ranks}) | {_lib.MECH_NAMES[b['mech']]} | "
                     f"{place.get(b['agent_kernel'], '?') if agent else '-'} | "
                     f"{('TMA (tile push)' if b['agent_kernel'] == 2 else 'TMA' if b['push'] == 1 else 'VEC16') if agent else '-'} | {b['chunk_bytes']} | "
                     f"{b['agent_warps'] if agent and b['agent_kernel'] != 2 else '-'} | {ms:.3f} |")
    txt = "\n".join(lines) + f"\n\nspace: `{SPACE}`\n"
    print(txt)
    if args.out:
        open(args.out, "w").write("# Profiler choices (Table II analogue), loopback on one B200\n\n" + txt)


if __name__ == "__main__":
    main()
