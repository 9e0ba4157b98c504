"""NEXT-1: ablation and cache-limit sweep on B200.

The paper's own variants: Fig. 6's ablation (memoization -> + dedup -> + time-encoding
precompute) and Table 4's cache-limit sweep {1e4, 1e5, 1e6, 3e6} (P:L450-466,
plus the 2e6 default of P:L380). Each row is cold-cache chronological passes over a whole
stream through tg_score_stream (the bench launch configuration: tf32x3 GEMMs,
default superbatch), device-timed with CUDA events, L2 flushed before each pass; edges/s is the
median of --passes passes. Outputs do not depend on the toggles (bit-exact invariance is a
GPU test), so only speed and the counters move.

    python tools/sweep.py [--configs reddit lastfm] [--passes 3] [--out profiles/.../sweep.json]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(s, flat, mc, opts, limit, passes, prec):
    import torch
    from paper_conf_ppopp_wangm23_b200 import Context, TG_NCOUNTERS
    ctx = Context.from_stream(s, device=0)
    ctx.load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                   max_batch_targets=2 * mc.batch, cache_limit=int(limit), time_window=mc.time_window,
                   opts=opts, precision=prec)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    src, dst, ts = d(s.src), d(s.dst), d(s.ts.view(np.int32))
    E = s.n_edges
    nb = (E + mc.batch - 1) // mc.batch
    sc = torch.zeros(E, dtype=torch.float32, device="cuda")
    log = torch.zeros(nb * TG_NCOUNTERS, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    st = torch.cuda.current_stream()
    ms = []
    for i in range(passes + 1):  # first pass = warm-up
        flush.zero_()
        ctx.cache_reset()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        ctx.score_stream(src, dst, ts, mc.batch, sc, log, stream=st)
        b.record(st)
        torch.cuda.synchronize()
        if i:
            ms.append(a.elapsed_time(b))
    c = ctx.counters()
    from paper_conf_ppopp_wangm23_b200 import counters_dict
    per = [counters_dict(r, mc.n_layers) for r in log.cpu().numpy().reshape(nb, TG_NCOUNTERS)]
    hit_b = [p["l1_hits"] / p["l1_lookups"] for p in per if p["l1_lookups"]]
    win = [sum(p["l1_hits"] for p in per[i:i + 10]) / max(1, sum(p["l1_lookups"] for p in per[i:i + 10]))
           for i in range(0, nb, 10)]
    med = float(np.median(ms))
    row = {
        "edges_per_s": E / (med / 1e3), "ms_per_pass": med, "ms_all": ms,
        "l1_hit_rate_mean_of_batches": float(np.mean(hit_b)) if hit_b else None,
        "l1_hit_rate_global": c["l1_hits"] / c["l1_lookups"] if c["l1_lookups"] else None,
        "l1_hit_rate_10batch_window_min": float(np.min(win)) if c["l1_lookups"] else None,
        "l1_hit_rate_10batch_window_max": float(np.max(win)) if c["l1_lookups"] else None,
        "computed": {f"l{l}": c[f"l{l}_misses"] for l in range(1, mc.n_layers + 1)},
        "evicted": c["l1_evicted"],
        "hit_rate_global_per_layer": {f"l{l}": (c[f"l{l}_hits"] / c[f"l{l}_lookups"] if c[f"l{l}_lookups"] else None)
                                      for l in range(1, mc.n_layers)},
        "time_table_hit_rate": c["t_table"] / max(1, c["t_table"] + c["t_direct"]),
        "cache_items_end": min(int(limit), c["l1_misses"]) if opts & 2 else 0,
        "cache_payload_mib_end": min(int(limit), c["l1_misses"]) * 4 * s.d_n / 2 ** 20 if opts & 2 else 0,
    }
    ctx.close()
    return row, sc.cpu().numpy()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", nargs="+", default=["reddit", "lastfm"])
    ap.add_argument("--passes", type=int, default=3)
    ap.add_argument("--precision", type=int, default=1)  # TG_PREC_TF32X3 (the bench headline)
    ap.add_argument("--out", default=None)
    ap.add_argument("--model", default=None, help="L,k override, e.g. 3,8 (NEXT-4: L = 3, k = 8)")
    args = ap.parse_args()
    over = {}
    if args.model:
        L, k = (int(v) for v in args.model.split(","))
        over = dict(n_layers=L, n_neighbors=k)
    from synth import get_config, make_stream, make_params
    D, C, T = 1, 2, 4  # TG_OPT_DEDUP, TG_OPT_CACHE, TG_OPT_TTABLE
    ablation = [("none", 0), ("cache", C), ("cache+dedup", C | D), ("cache+dedup+ttable", C | D | T)]
    limits = [10_000, 100_000, 1_000_000, 2_000_000, 3_000_000]
    res = []
    for name in args.configs:
        cfg = get_config(name, **over)
        mc = cfg.model
        s = make_stream(name)
        flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
        ref = None
        for label, opts in ablation:
            row, sc = run(s, flat, mc, opts, mc.cache_limit, args.passes, args.precision)
            if ref is None:
                ref = sc
            row.update(config=name, model=f"L{mc.n_layers}k{mc.n_neighbors}", sweep="ablation", opts=label, cache_limit=mc.cache_limit,
                       scores_equal_to_none=bool(np.array_equal(sc, ref)))
            print(json.dumps(row), flush=True)
            res.append(row)
        for lim in limits:
            row, sc = run(s, flat, mc, C | D | T, lim, args.passes, args.precision)
            row.update(config=name, model=f"L{mc.n_layers}k{mc.n_neighbors}", sweep="cache_limit", opts="cache+dedup+ttable", cache_limit=lim,
                       scores_equal_to_none=bool(np.array_equal(sc, ref)))
            print(json.dumps(row), flush=True)
            res.append(row)
    if args.out:
        os.makedirs(os.path.dirname(args.out), exist_ok=True)
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
