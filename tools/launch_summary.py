"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel.

    python tools/launch_summary.py launches.csv [--json out.json]
"""
import csv
import json
import sys


def summarise(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.DictReader(lines[start:]))
    k = {}
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        u = r["Metric Unit"]
        v = v / 1e3 if u == "nsecond" or u == "ns" else v * 1e3 if u in ("msecond", "ms") else v
        name = r["Kernel Name"].split("(")[0]
        d = k.setdefault(name, {"launches": 0, "total_us": 0.0})
        d["launches"] += 1
        d["total_us"] += v
    tot = sum(d["total_us"] for d in k.values())
    out = {}
    for n, d in sorted(k.items(), key=lambda kv: -kv[1]["total_us"]):
        out[n] = {"launches": d["launches"], "total_ms": round(d["total_us"] / 1e3, 3),
                  "share": round(d["total_us"] / tot, 4), "avg_us": round(d["total_us"] / d["launches"], 2)}
    return {"total_ms": round(tot / 1e3, 3), "kernels": out}


if __name__ == "__main__":
    s = summarise(sys.argv[1])
    if "--json" in sys.argv:
        json.dump(s, open(sys.argv[sys.argv.index("--json") + 1], "w"), indent=1)
    print(json.dumps(s, indent=1))
