"""Error statistics of the GPU path vs the plain oracle at the bench configuration.

Whole Reddit-shaped stream through tg_score_stream (bench launch config, cold cache), then
tg_embed_batch on the src || dst targets of stratified batches (warm cache: layer-1 rows come
from the stream pass). Prints, per precision, max |d|, max |d|/|ref|, and the smallest atol
that makes |d| <= atol + rtol |ref| hold at the north_star rtol -- the evidence behind the
tolerances written in tests/ and DESIGN.md (R17, R22).

    python tools/parity_errors.py [--config reddit] [--prec 1 2] [--out file.json]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests.gpu_helpers import setup, make_ctx, make_oracle  # noqa: E402

RTOL = {0: 1e-4, 1: 1e-4, 2: 2e-2, 3: 2e-2, 4: 1e-4}


def stats(got, ref, rtol):
    d = np.abs(got.astype(np.float64) - ref)
    need = np.maximum(d - rtol * np.abs(ref), 0.0)
    return {"max_abs": float(d.max()), "max_rel": float((d / np.maximum(np.abs(ref), 1e-30)).max()),
            "p999_abs": float(np.quantile(d, 0.999)), "atol_needed_at_rtol": float(need.max()),
            "ref_absmax": float(np.abs(ref).max()), "n": int(d.size)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="reddit")
    ap.add_argument("--prec", type=int, nargs="+", default=[1, 2])
    ap.add_argument("--batches", type=int, default=8)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    cfg, s, flat = setup(a.config)
    mc = cfg.model
    o = make_oracle(s, flat, mc)
    nb = (s.n_edges + mc.batch - 1) // mc.batch
    picks = sorted(set(np.linspace(0, nb - 1, a.batches).astype(int).tolist()))
    dev = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
    refs = {}
    for b in picks:
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        refs[b] = o.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
    res = {"config": a.config, "batches": picks}
    for prec in a.prec:
        ctx = make_ctx(s, flat, mc, precision=prec)
        sc = torch.zeros(s.n_edges, dtype=torch.float32, device="cuda")
        ctx.score_stream(dev(s.src), dev(s.dst), dev(s.ts.view(np.int32)), mc.batch, sc)
        torch.cuda.synchronize()
        scores = sc.cpu().numpy()
        ge, re_, gs, rs = [], [], [], []
        for b in picks:
            lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
            nodes = np.r_[s.src[lo:hi], s.dst[lo:hi]].astype(np.int32)
            ts = np.r_[s.ts[lo:hi], s.ts[lo:hi]].astype(np.uint32)
            out = torch.zeros(nodes.size * s.d_n, dtype=torch.float32, device="cuda")
            ctx.embed_batch(dev(nodes), dev(ts.view(np.int32)), out)
            torch.cuda.synchronize()
            ge.append(out.cpu().numpy().reshape(nodes.size, s.d_n))
            re_.append(refs[b][0])
            gs.append(scores[lo:hi])
            rs.append(refs[b][1])
        res[f"prec{prec}"] = {"embed": stats(np.concatenate(ge), np.concatenate(re_), RTOL[prec]),
                              "score": stats(np.concatenate(gs), np.concatenate(rs), RTOL[prec]),
                              "superbatch": ctx.superbatch()}
        ctx.close()
        print(prec, json.dumps(res[f"prec{prec}"]), flush=True)
    if a.out:
        json.dump(res, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
