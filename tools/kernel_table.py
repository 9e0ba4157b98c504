"""Per-kernel roofline table from one `ncu --set full` capture of a superbatch's launches.

For every captured launch: duration, DRAM bytes (read + write), achieved DRAM GB/s and its
fraction of the measured HBM peak (MEASURED_PEAKS.json), L2 hit rate, tensor-pipe activity
(% of peak while active), warps active, registers. GEMM launches are labelled G1..G4 / score
by their position in the layer chain. Writes markdown + JSON.

    python tools/kernel_table.py report.ncu-rep --out profiles/r02/kernels_tf32x3 [--tag tf32x3]
"""
import argparse
import json
import os
import re
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summarise  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--out", required=True)
    ap.add_argument("--tag", default="")
    a = ap.parse_args()
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    hbm = peaks["hbm_gbs"]
    rows = []
    # GEMM role from its predecessor in the layer chain: G1 precedes the
    # attention, G2 follows it, G3 follows the LayerNorm, G4 follows G3, score follows k_score_rows
    prev_role = {"k_attn_g": "G2", "k_attn": "G2", "k_layernorm": "G3", "G3": "G4", "k_score_rows": "score"}
    prev = ""
    for lid, d in sorted(summarise(a.rep).items(), key=lambda kv: int(kv[0])):
        name = re.sub(r"\(.*", "", d["kernel"]).replace("void ", "").replace("tg::", "").strip()
        base = re.sub(r"<.*", "", name)
        if base in ("k_gemm_tc", "k_gemm_simt"):
            role = prev_role.get(prev, "G1")
            name = f"{name} {role}"
            prev = role
        else:
            prev = base
        dur = d.get("dur_us", 0.0)
        rb, wb = d.get("dram__bytes_read.sum", 0.0), d.get("dram__bytes_write.sum", 0.0)
        gbs = (rb + wb) / (dur * 1e-6) / 1e9 if dur else 0.0
        rows.append({"id": int(lid), "kernel": name, "us": dur, "dram_MB": (rb + wb) / 1e6, "dram_GBs": gbs,
                     "dram_frac_of_peak": gbs / hbm, "l2_hit_pct": d.get("l2_hit_pct"),
                     "tensor_active_pct": d.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"),
                     "warps_active_pct": d.get("occ_pct"), "regs": d.get("regs"), "grid": d.get("grid"),
                     "ipc": d.get("ipc")})
    json.dump({"tag": a.tag, "hbm_peak_gbs": hbm, "launches": rows}, open(a.out + ".json", "w"), indent=1)
    with open(a.out + ".md", "w") as f:
        f.write(f"# ncu --set full, one superbatch {a.tag} (HBM peak {hbm} GB/s measured)\n\n")
        f.write("| kernel | us | DRAM MB | DRAM GB/s | of HBM peak | L2 hit % | tensor active % | warps active % | regs |\n")
        f.write("|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            ta = r["tensor_active_pct"]
            f.write(f"| {r['kernel']} | {r['us']:.1f} | {r['dram_MB']:.1f} | {r['dram_GBs']:.0f} | "
                    f"{r['dram_frac_of_peak']:.2f} | {r['l2_hit_pct'] or 0:.0f} | "
                    f"{'' if ta is None else f'{ta:.0f}'} | {r['warps_active_pct'] or 0:.0f} | {r['regs'] or 0:.0f} |\n")
    print(open(a.out + ".md").read())


if __name__ == "__main__":
    main()
