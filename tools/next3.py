"""NEXT-3: link-prediction evaluation with negatives on B200, superbatched.

Each chronological batch of B edges embeds src || dst || neg at the edge times as ONE
deduplicated target list (3B = 600 targets; TGAT's evaluation [37]) and scores
the positive pairs (src, dst) and the negative pairs (src, neg) -- through tg_score_stream_neg,
the same superbatched two-stream path as the positive-only stream. Negatives come from the
seeded uniform sampler over the stream's destination nodes (synth.negatives, an input).
Device buffers, cold cache per pass, L2 flushed, CUDA events; reports edges/s, hit rates, and
AP / AUC of the whole stream (the random-weight model ranks near chance: AP/AUC are reported
to show the evaluation runs end to end; their parity with the oracle is pinned in
tests/test_gpu_fullsize.py::test_stream_negatives_parity_ap_auc).

    python tools/next3.py [--config reddit] [--precision tf32x3] [--out profiles/.../next3.json]
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
    ap.add_argument("--precision", default="tf32x3")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    from sklearn.metrics import average_precision_score, roc_auc_score
    from synth import make_stream, make_params, negatives, get_config
    from paper_conf_ppopp_wangm23_b200 import Context, TG_NCOUNTERS, counters_dict
    from paper_conf_ppopp_wangm23_b200 import tg as tgm
    prec = {"fp32": 0, "tf32x3": 1, "bf16": 2, "tf32": 3, "f16x3": 4}[a.precision]
    cfg = get_config(a.config)
    mc = cfg.model
    s = make_stream(a.config)
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    neg = negatives(s, seed=1)
    B = mc.batch
    E = s.n_edges
    nb = (E + B - 1) // B
    dev = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
    src, dst, ts, ng = dev(s.src), dev(s.dst), dev(s.ts.view(np.int32)), dev(neg)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    out = {"config": a.config, "precision": a.precision, "n_edges": E, "batch": B}
    for mode in ("with_negatives", "positives_only"):
        ctx = Context.from_stream(s, device=0)
        ctx.load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                       max_batch_targets=3 * B, cache_limit=mc.cache_limit, time_window=mc.time_window,
                       precision=prec)
        scores = torch.zeros(2 * E, dtype=torch.float32, device="cuda")
        log = torch.zeros(nb * TG_NCOUNTERS, dtype=torch.int64, device="cuda")

        def run():
            ctx.cache_reset()
            if mode == "with_negatives":
                ctx.score_stream_neg(src, dst, ts, ng, B, scores, log)
            else:
                ctx.score_stream(src, dst, ts, B, scores[:E], log)

        for _ in range(2):
            run()
        ms = []
        for _ in range(a.steps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            run()
            e1.record()
            torch.cuda.synchronize()
            ms.append(e0.elapsed_time(e1))
        c = ctx.counters()
        r = {"ms_per_pass": float(np.median(ms)), "edges_per_s": E / (float(np.median(ms)) / 1e3),
             "superbatch": ctx.superbatch(), "l1_hit_rate": c["l1_hits"] / max(1, c["l1_lookups"]),
             "l1_lookups": c["l1_lookups"], "computed": {f"l{l}": c[f"l{l}_misses"] for l in (1, 2)},
             "dedup_ratio_l2": 1 - c["l2_unique"] / max(1, c["l2_n"])}
        if mode == "with_negatives":
            sc = scores.cpu().numpy()
            y = np.r_[np.ones(E), np.zeros(E)]
            r["AP"] = float(average_precision_score(y, sc))
            r["AUC"] = float(roc_auc_score(y, sc))
        out[mode] = r
        print(mode, json.dumps(r), flush=True)
        ctx.close()
    if a.out:
        json.dump(out, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
