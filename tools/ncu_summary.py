"""Summarise an .ncu-rep: one line per profiled launch with the key metrics.

    python tools/ncu_summary.py report.ncu-rep [--json out.json]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = {
    "Duration": "dur_us",
    "DRAM Throughput": "dram_pct",
    "Memory Throughput": "mem_pct",
    "L2 Cache Throughput": "l2_pct",
    "Compute (SM) Throughput": "sm_pct",
    "Executed Ipc Active": "ipc",
    "Achieved Occupancy": "occ_pct",
    "Registers Per Thread": "regs",
    "Grid Size": "grid",
    "Block Size": "block",
    "L2 Hit Rate": "l2_hit_pct",
    "Executed Instructions": "instr",
}


def summarise(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[0]
    ix = {h: i for i, h in enumerate(hdr)}
    launches = {}
    for r in rows[1:]:
        if len(r) <= ix["Metric Value"]:
            continue
        lid = r[ix["ID"]]
        d = launches.setdefault(lid, {"kernel": r[ix["Kernel Name"]][:60]})
        m = r[ix["Metric Name"]]
        if m in KEYS:
            v = r[ix["Metric Value"]].replace(",", "")
            unit = r[ix["Metric Unit"]]
            try:
                v = float(v)
            except ValueError:
                pass
            if m == "Duration" and unit == "ms":
                v *= 1e3
            if m == "Duration" and unit == "ns":
                v /= 1e3
            d[KEYS[m]] = v
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(io.StringIO(raw)))
    if len(rr) > 2:
        h = rr[0]
        want = [c for c in h if c in ("dram__bytes_read.sum", "dram__bytes_write.sum",
                                       "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
                                       "sm__inst_executed_pipe_tensor_op_hmma.avg.pct_of_peak_sustained_active")
                or c.startswith("sm__pipe_tensor")]
        units = rr[1]
        for row in rr[2:]:
            lid = row[h.index("ID")]
            d = launches.get(lid)
            if d is None:
                continue
            for c in want:
                i = h.index(c)
                try:
                    v = float(row[i].replace(",", ""))
                except ValueError:
                    continue
                u = units[i]
                if u == "Kbyte":
                    v *= 1e3
                elif u == "Mbyte":
                    v *= 1e6
                elif u == "Gbyte":
                    v *= 1e9
                d[c] = v
    return launches


if __name__ == "__main__":
    res = summarise(sys.argv[1])
    for lid, d in res.items():
        print(lid, json.dumps(d))
    if "--json" in sys.argv:
        json.dump(res, open(sys.argv[sys.argv.index("--json") + 1], "w"), indent=1)
