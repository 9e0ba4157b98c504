"""Hottest SASS instructions of an ncu source-page CSV (--page source --csv --print-source sass).

    python tools/sass_hot.py src.csv[.gz] [--top 40] [--context 0]
Prints per instruction: all samples, wait / short_sb / long_sb / branch samples, the instruction.
"""
import argparse
import csv
import gzip
import io


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--top", type=int, default=40)
    ap.add_argument("--listing", action="store_true", help="print every instruction in address order")
    a = ap.parse_args()
    op = gzip.open if a.csv.endswith(".gz") else open
    lines = io.TextIOWrapper(op(a.csv, "rb"), "utf-8").read().splitlines()
    rows = list(csv.reader(lines[1:]))
    hdr, body = rows[0], rows[1:]
    ix = {h: i for i, h in enumerate(hdr)}
    cols = ["Warp Stall Sampling (All Samples)", "stall_wait", "stall_short_sb", "stall_long_sb",
            "stall_branch_resolving", "stall_selected"]
    recs = []
    for n, r in enumerate(body):
        try:
            v = [int(r[ix[c]]) for c in cols]
        except (ValueError, IndexError, KeyError):
            continue
        recs.append((n, v, r[ix["Source"]].strip()))
    tot = sum(v[0] for _, v, _ in recs)
    print(f"total samples {tot}; columns: all wait short_sb long_sb branch selected")
    sel = recs if a.listing else sorted(recs, key=lambda x: -x[1][0])[:a.top]
    for n, v, s in sel:
        print(f"{n:5d} {v[0]:6d} {v[1]:5d} {v[2]:5d} {v[3]:5d} {v[4]:5d} {v[5]:5d}  {s}")


if __name__ == "__main__":
    main()
