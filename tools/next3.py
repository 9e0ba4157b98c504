"""NEXT-3: link-prediction evaluation with negatives on B200.

Each chronological batch of B edges embeds src || dst || neg at the edge times as one
deduplicated target list (3B = 600 targets; TGAT's evaluation [37]) and scores
the positive pairs (src, dst) and the negative pairs (src, neg) through tg_score_pairs.
Negatives come from a seeded uniform sampler over the destination nodes of the stream.
One call per batch (no superbatching yet), device buffers, cold cache, CUDA-event timed over
the whole stream after one warm-up pass; reports edges/s, and the counters (AP/AUC are
not computed: the synthetic weights carry no signal).

    python tools/next3.py [--config reddit] [--n-edges N] [--out profiles/.../next3.json]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="reddit")
    ap.add_argument("--n-edges", type=int, default=None)
    ap.add_argument("--prec", type=int, default=2)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    from synth.configs import get_config
    from synth import make_stream, make_params
    from paper_conf_ppopp_wangm23_b200 import Context
    cfg = get_config(a.config)
    mc = cfg.model
    s = make_stream(a.config, n_edges=a.n_edges)
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    B = mc.batch
    ctx = Context.from_stream(s, device=0)
    ctx.load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                   max_batch_targets=3 * B, cache_limit=mc.cache_limit, time_window=mc.time_window,
                   precision=a.prec)
    E = s.n_edges
    nb = (E + B - 1) // B
    rng = np.random.default_rng(7)
    dst_pool = np.unique(s.dst)
    neg = dst_pool[rng.integers(0, dst_pool.size, E)].astype(np.int32)
    nodes = np.empty(3 * E, np.int32)
    tts = np.empty(3 * E, np.uint32)
    pa = np.empty(2 * E, np.int32)
    pb = np.empty(2 * E, np.int32)
    offs = []
    for b in range(nb):
        lo, hi = b * B, min(E, (b + 1) * B)
        n = hi - lo
        o = 3 * lo
        nodes[o:o + 3 * n] = np.concatenate([s.src[lo:hi], s.dst[lo:hi], neg[lo:hi]])
        tts[o:o + 3 * n] = np.tile(s.ts[lo:hi], 3)
        pa[2 * lo:2 * hi] = np.concatenate([np.arange(n), np.arange(n)])
        pb[2 * lo:2 * hi] = np.concatenate([n + np.arange(n), 2 * n + np.arange(n)])
        offs.append((lo, n))
    d = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
    dn, dt, da, db = d(nodes), d(tts.view(np.int32)), d(pa), d(pb)
    out = torch.zeros(2 * E, dtype=torch.float32, device="cuda")
    st = torch.cuda.current_stream()
    times = []
    for rep in range(2):  # first pass = warm-up
        ctx.cache_reset()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for lo, n in offs:
            ctx.score_pairs(dn[3 * lo:3 * lo + 3 * n], dt[3 * lo:3 * lo + 3 * n], da[2 * lo:2 * lo + 2 * n],
                            db[2 * lo:2 * lo + 2 * n], out[2 * lo:2 * lo + 2 * n], stream=st)
        e1.record(st)
        torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    c = ctx.counters()
    res = {"config": a.config, "n_edges": E, "batch": B, "targets_per_batch": 3 * B, "prec": a.prec,
           "ms": times[-1], "edges_per_sec": E / (times[-1] / 1e3), "counters": c,
           "scores_finite": bool(torch.isfinite(out).all().item())}
    print(json.dumps(res))
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
