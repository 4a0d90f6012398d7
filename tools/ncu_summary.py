"""Summarise an ncu report (run here, no GPU): key metrics + top stall reasons -> JSON + Markdown.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep profiles/r01_jacobi  [alg_bytes_per_launch]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "sm__cycles_elapsed.avg.per_second"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6,
         "ms": 1e-3, "msecond": 1e-3, "nsecond": 1e-9}


def main():
    rep, out = sys.argv[1], sys.argv[2]
    alg = float(sys.argv[3]) if len(sys.argv) > 3 else None
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, u = rows[0], rows[1]
    res = []
    for v in rows[2:]:
        d = {"kernel": v[h.index("Kernel Name")]}
        for k in KEYS:
            if k in h:
                i = h.index(k)
                try:
                    d[k] = float(v[i].replace(",", ""))
                except ValueError:
                    d[k] = v[i]
                d[k + ".unit"] = u[i]
        st = []
        for i, n in enumerate(h):
            if "smsp__pcsamp_warps_issue_stalled" in n and not n.endswith("not_issued"):
                try:
                    st.append((float(v[i]), n.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
        tot = sum(x for x, _ in st) or 1.0
        d["top_stalls"] = [[n, round(x / tot, 3)] for x, n in sorted(st, reverse=True)[:6]]
        rb = d.get("dram__bytes_read.sum", 0) * SCALE.get(d.get("dram__bytes_read.sum.unit", "byte"), 1)
        wb = d.get("dram__bytes_write.sum", 0) * SCALE.get(d.get("dram__bytes_write.sum.unit", "byte"), 1)
        d["dram_bytes_per_launch"] = rb + wb
        t = d.get("gpu__time_duration.sum", 0) * SCALE.get(d.get("gpu__time_duration.sum.unit", "ns"), 1e-9)
        d["duration_s"] = t
        if t:
            d["dram_GBps"] = (rb + wb) / t / 1e9
        if alg:
            d["alg_bytes_per_launch"] = alg
            d["traffic_over_alg"] = (rb + wb) / alg
        res.append(d)
    json.dump(res[0] if len(res) == 1 else res, open(out + ".json", "w"), indent=1)
    with open(out + ".md", "w") as f:
        for d in res:
            f.write(f"### {d['kernel'][:100]}\n\n| metric | value |\n|---|---|\n")
            for k in KEYS + ["dram_bytes_per_launch", "duration_s", "dram_GBps", "alg_bytes_per_launch",
                             "traffic_over_alg"]:
                if k in d:
                    f.write(f"| {k} | {d[k]} {d.get(k + '.unit', '')} |\n")
            f.write(f"| top stalls | {d['top_stalls']} |\n\n")
    print(open(out + ".md").read())


if __name__ == "__main__":
    main()
