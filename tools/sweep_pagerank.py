"""PageRank phase-kernel time on RMAT-SCALE for library variants x hot-table sizes.

    python tools/sweep_pagerank.py VARIANT_LIB[,LIB2...] HOT[,HOT2...]
Each (lib, hot) runs in a fresh process (PROACT_LIB / PROACT_GRAPH_HOT), prints one line.
"""
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def one():
    os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
    sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    import synth
    from paper_conf_isca_muthukrishnannl21_b200 import _lib
    from paper_conf_isca_muthukrishnannl21_b200 import runtime as rt
    from paper_conf_isca_muthukrishnannl21_b200 import workloads as wl
    scale = int(os.environ.get("SCALE", 24))
    torch.cuda.set_device(0)
    rt.init(1, 0, rt.new_job_key())
    cache = f"/tmp/rmat{scale}.npz"   # generated once per box by the first run
    if os.path.exists(cache):
        z = np.load(cache)
        src, dst = z["src"], z["dst"]
    else:
        src, dst = synth.rmat(scale, 16)
        np.savez(cache, src=src, dst=dst)
    V = 1 << scale
    if os.environ.get("RELABEL"):   # experiment: ids by descending out-degree (stable)
        od = np.bincount(src, minlength=V)
        order = np.argsort(-od, kind="stable")
        new = np.empty(V, np.uint32)
        new[order] = np.arange(V, dtype=np.uint32)
        src, dst = new[src], new[dst]
    s = torch.cuda.Stream()
    P = wl.PageRank(V, src, dst, 131072, stream=s)
    ts = []
    for k in range(14):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        i = P.k & 1
        a.record(s)
        _lib.check(rt.lib().proact_pagerank_phase(P.gid, P.rid[i], P.rid[i ^ 1], P.d, wl._s(s)), "pr")
        b.record(s)
        rt.phase_sync(s)
        P.k += 1
        ts.append((a, b))
    torch.cuda.synchronize()
    pr = statistics.median(a.elapsed_time(b) for a, b in ts[3:])
    print(f"relabel={os.environ.get('RELABEL', '')} lib={os.environ.get('PROACT_LIB', 'default')} hot={os.environ.get('PROACT_GRAPH_HOT', '-')} "
          f"kernel={os.environ.get('PROACT_PR_KERNEL', 'hot')} nhot={P.nhot}: pagerank {pr:.4f} ms", flush=True)
    P.free()
    rt.finalize()


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--one":
        one()
        sys.exit(0)
    libs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["default"]
    hots = sys.argv[2].split(",") if len(sys.argv) > 2 else ["-1"]
    for lib in libs:
        for h in hots:
            env = dict(os.environ)
            if lib != "default":
                env["PROACT_LIB"] = lib
            if h == "plain":
                env["PROACT_PR_KERNEL"] = "plain"
                env["PROACT_GRAPH_HOT"] = "0"
            elif h != "-1":
                env["PROACT_GRAPH_HOT"] = h
            subprocess.run([sys.executable, os.path.abspath(__file__), "--one"], env=env, timeout=600)
