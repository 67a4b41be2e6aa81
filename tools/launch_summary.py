"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into per-kernel launches, total,
average and share of the GPU time: python tools/launch_summary.py launches.csv "<command>" > summary.json"""
import csv
import json
import sys


def main():
    path = sys.argv[1]
    src = sys.argv[2] if len(sys.argv) > 2 else ""
    rows = []
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    for r in csv.DictReader(lines):
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        if r["Metric Unit"] == "us":
            v *= 1e3
        elif r["Metric Unit"] == "ms":
            v *= 1e6
        rows.append((r["Kernel Name"], v))
    tot = sum(v for _, v in rows)
    agg = {}
    for k, v in rows:
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += v
    out = {"source": src, "kernels": {}}
    for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out["kernels"][k] = {"launches": c, "total_us": round(t / 1e3, 1), "avg_us": round(t / c / 1e3, 2),
                             "share": round(t / tot, 4)}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
