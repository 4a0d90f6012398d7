"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) as a Markdown table.

    python tools/launch_summary.py gpurun_out/launches.csv "<the profiled command>" > profiles/rNN_launches.md
"""
import collections
import csv
import re
import sys


def main():
    path, cmd = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.DictReader(lines))
    agg = collections.OrderedDict()
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = re.sub(r"\(.*", "", r["Kernel Name"]).replace("void ", "").replace("<unnamed>::", "")
        t = float(r["Metric Value"]) * {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3,
                                          "ms": 1e3, "msecond": 1e3}.get(r["Metric Unit"], 1.0)
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += t
    tot = sum(v[1] for v in agg.values())
    print(f"# ncu launch list of `{cmd}`\n")
    print("`ncu --metrics gpu__time_duration.sum --clock-control none` -- cold-cache, serialised: compare SHARES.\n")
    print("| kernel | launches | total us | share | mean us |")
    print("|---|---|---|---|---|")
    for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"| {k} | {n} | {t:.1f} | {t / tot:.3f} | {t / n:.2f} |")


if __name__ == "__main__":
    main()
