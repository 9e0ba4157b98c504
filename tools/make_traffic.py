"""profiles/traffic.json: measured DRAM bytes per launch of each bench kernel, from a committed
`ncu --set full` superbatch capture (tools/kernel_table.py JSON), stamped with its provenance.

    python tools/make_traffic.py profiles/r02/kernels_tf32x3.json --config reddit --prec tf32x3 \
        --superbatch 64 --targets-per-launch 25354 --build <git sha>
"""
import argparse
import collections
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("table")
    ap.add_argument("--config", default="reddit")
    ap.add_argument("--prec", default="tf32x3")
    ap.add_argument("--superbatch", type=int, required=True)
    ap.add_argument("--targets-per-launch", type=float, required=True)
    ap.add_argument("--build", default="")
    a = ap.parse_args()
    rows = json.load(open(a.table))["launches"]
    agg = collections.defaultdict(list)
    for r in rows:
        k = r["kernel"]
        if k.startswith("k_attn_g"):
            k = "k_attn_g"
        elif k.startswith("k_gemm_tc"):
            k = "k_gemm_tc " + k.split()[-1]
        agg[k].append(r)
    out_path = os.path.join(ROOT, "profiles", "traffic.json")
    doc = json.load(open(out_path)) if os.path.exists(out_path) else {}
    rec = {}
    for k, v in agg.items():
        rec[k] = {"dram_bytes_per_launch": sum(x["dram_MB"] for x in v) / len(v) * 1e6,
                  "ncu_us_per_launch": sum(x["us"] for x in v) / len(v), "launches_captured": len(v),
                  "superbatch": a.superbatch, "targets_per_launch": a.targets_per_launch,
                  "source": os.path.relpath(a.table, ROOT), "build": a.build}
    doc.setdefault(a.config, {})[a.prec] = rec
    json.dump(doc, open(out_path, "w"), indent=1)
    print(json.dumps({k: round(v["dram_bytes_per_launch"] / 1e6, 1) for k, v in rec.items()}))


if __name__ == "__main__":
    main()
