"""Print one superbatch's kernel launches (name, grid, us) from an ncu --csv launch list,
plus the per-kernel average over the whole list.

    python tools/sb_launches.py launches.csv
"""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr]
ik, ig, iv = h.index("Kernel Name"), h.index("Grid Size"), h.index("Metric Value")
im = h.index("Metric Name") if "Metric Name" in h else None
L = []
for r in rows[hdr + 1:]:
    if len(r) > iv and (im is None or r[im] == "gpu__time_duration.sum"):  # one row per launch
        name = re.sub(r"\(.*", "", r[ik]).replace("void ", "").replace("tg::", "")
        L.append((name, r[ig], float(r[iv]) / 1e3))
starts = [i for i, x in enumerate(L) if x[0] == "k_dedup"]
if len(starts) >= 4:
    a, b = starts[1], starts[3]  # two dedup launches per superbatch (levels L and L-1)
    tot = 0.0
    for n, g, us in L[a:b]:
        print(f"  {n:28s} {g:14s} {us:8.2f}")
        tot += us
    print(f"  superbatch serialized total {tot:.1f} us")
agg = collections.defaultdict(list)
for n, g, us in L:
    agg[n].append(us)
for n, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{n:28s} n={len(v):4d} avg={sum(v)/len(v):8.2f} us total={sum(v)/1e3:8.3f} ms")
