"""NEXT-2: host-resident vs device-resident memo cache on B200.

The paper's GPU design keeps TGOpt's cache in host RAM and reports the host<->device copy
share of GPU activity (Table 5), adding that "this can change
given a different design". Here the same hot path runs with the FIFO payload ring of the
cached layer either in HBM (default) or in pinned, mapped host memory (TG_OPT_HOST_CACHE,
index in HBM); kernels read/write the ring rows directly over the host link. Reported per
stream and location: edges/s (cold-cache pass, CUDA events, median of K), hit rate, and the
algorithmic bytes that cross the host link per pass, from the counters: writes of every
computed layer-1 embedding (l1_misses x d_n x 4) and reads of the cached rows the layer-2
computations gather (l2_misses x (k + 1) x d_n x 4 for the attention's neighbour and target
rows, + l2_misses x d_n x 4 for the target row of the merge FFN).

    python tools/next2.py [--configs reddit lastfm] [--precision tf32x3] [--out file.json]
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
    ap.add_argument("--configs", nargs="+", default=["reddit", "lastfm"])
    ap.add_argument("--precision", default="tf32x3")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    from synth import make_stream, make_params, get_config
    from paper_conf_ppopp_wangm23_b200 import Context, TG_OPT_ALL, TG_OPT_HOST_CACHE
    prec = {"fp32": 0, "tf32x3": 1, "bf16": 2, "tf32": 3, "f16x3": 4}[a.precision]
    res = {"precision": a.precision, "runs": []}
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    for name in a.configs:
        cfg = get_config(name)
        mc = cfg.model
        s = make_stream(name)
        flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
        dev = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
        src, dst, ts = dev(s.src), dev(s.dst), dev(s.ts.view(np.int32))
        ref = None
        for where, opts in (("device", TG_OPT_ALL), ("host", TG_OPT_ALL | TG_OPT_HOST_CACHE)):
            ctx = Context.from_stream(s, device=0)
            ctx.load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                           max_batch_targets=2 * mc.batch, cache_limit=mc.cache_limit,
                           time_window=mc.time_window, precision=prec, opts=opts)
            sc = torch.zeros(s.n_edges, dtype=torch.float32, device="cuda")
            ms = []
            for it in range(a.steps + 1):
                flush.zero_()
                ctx.cache_reset()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                ctx.score_stream(src, dst, ts, mc.batch, sc)
                e1.record()
                torch.cuda.synchronize()
                if it:
                    ms.append(e0.elapsed_time(e1))
            c = ctx.counters()
            k, dn = mc.n_neighbors, s.d_n
            wr = c["l1_misses"] * dn * 4
            rd = c["l2_misses"] * (k + 2) * dn * 4
            scores = sc.cpu().numpy()
            if ref is None:
                ref = scores
            t = float(np.median(ms))
            r = {"config": name, "cache": where, "ms_per_pass": t, "edges_per_s": s.n_edges / (t / 1e3),
                 "l1_hit_rate": c["l1_hits"] / max(1, c["l1_lookups"]), "evicted": c["l1_evicted"],
                 "host_link_bytes_per_pass": (wr + rd) if where == "host" else 0,
                 "cache_payload_bytes_per_pass": wr + rd,
                 "effective_host_link_gbs": ((wr + rd) / (t / 1e3) / 1e9) if where == "host" else None,
                 "max_abs_score_diff_vs_device": float(np.abs(scores - ref).max()),
                 "superbatch": ctx.superbatch()}
            res["runs"].append(r)
            print(json.dumps(r), flush=True)
            ctx.close()
    if a.out:
        json.dump(res, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
