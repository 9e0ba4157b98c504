"""Per-CUDA-line instruction / stall-sample breakdown of one kernel in an .ncu-rep.

    python tools/ncu_lines.py report.ncu-rep [--top 30] [--kernel regex]
"""
import argparse
import collections
import csv
import io
import subprocess

ap = argparse.ArgumentParser()
ap.add_argument("rep")
ap.add_argument("--top", type=int, default=30)
ap.add_argument("--sort", default="samples")
a = ap.parse_args()
out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
h = rows[hi]
ix = {}
for i, k in enumerate(h):
    ix.setdefault(k, i)
src_of = {}
agg = collections.defaultdict(lambda: collections.Counter())
line = None
stalls = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]


def f(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


for r in rows[hi + 1:]:
    if len(r) < len(h):
        continue
    if r[0] == "Line No":
        continue
    if r[0]:
        line = int(r[0])
        src_of[line] = r[1].strip()
    if not r[2]:
        continue
    c = agg[line]
    c["instr"] += f(r[ix["Instructions Executed"]])
    c["samples"] += f(r[ix["Warp Stall Sampling (All Samples)"]])
    for s in stalls:
        c[s[6:]] += f(r[h.index(s)])
ti = sum(c["instr"] for c in agg.values())
ts = sum(c["samples"] for c in agg.values())
print(f"instructions {ti:.0f}  samples {ts:.0f}")
for ln, c in sorted(agg.items(), key=lambda kv: -kv[1][a.sort])[:a.top]:
    top = sorted(((v, k) for k, v in c.items() if k not in ("instr", "samples")), reverse=True)[:3]
    print(f"{ln:5d} {100 * c['instr'] / ti:5.1f}%i {100 * c['samples'] / ts:5.1f}%s  {src_of.get(ln, '')[:64]:64s} "
          + " ".join(f"{k}:{int(v)}" for v, k in top))
