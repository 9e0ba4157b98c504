"""Per-batch duplication of the plain TGAT batch expansion (Table 1) on a
synthetic stream -- the calibration target of synth/ (SURVEY 8(d)).

Definitions: the layer-L input is src || dst at the edge time; the layer-(l-1)
input is [layer-l input ; its k most-recent neighbours] with no dedup (the baseline TGAT); a
duplicate is an equal (node, t) pair, except at layer 0 where timestamps are irrelevant and
only the node id counts. Reported: mean over sampled batches of 1 - unique / n per layer.

    python tools/calibrate.py reddit [--batches 200] [--set p_rep=0.3 zipf_item=0.9 ...]
"""
import argparse
import dataclasses
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import make_stream, get_config  # noqa: E402


class CSR:
    def __init__(self, V, src, dst, ts):
        E = src.size
        node = np.concatenate([src, dst]).astype(np.int64)
        nbr = np.concatenate([dst, src]).astype(np.int64)
        eid = np.concatenate([np.arange(1, E + 1)] * 2)
        tt = np.concatenate([ts, ts]).astype(np.int64)
        o = np.lexsort((eid, tt, node))
        self.node, self.nbr, self.t = node[o], nbr[o], tt[o]
        self.key = self.node * (1 << 33) + self.t          # sorted (node, t)
        self.lo = np.searchsorted(self.node, np.arange(V + 2))

    def sample(self, nodes, ts, k):
        """most-recent k with t_j < t, right-aligned, padding (0, 0)"""
        nodes = nodes.astype(np.int64)
        p = np.searchsorted(self.key, nodes * (1 << 33) + ts.astype(np.int64), side="left")
        lo = self.lo[nodes]
        idx = p[:, None] - k + np.arange(k)[None, :]
        ok = idx >= lo[:, None]
        idx = np.where(ok, idx, 0)
        nb = np.where(ok, self.nbr[idx], 0)
        tj = np.where(ok, self.t[idx], 0)
        return nb, tj


def dup(nodes, ts=None):
    if ts is None:
        u = np.unique(nodes).size
    else:
        u = np.unique(nodes.astype(np.int64) * (1 << 33) + ts.astype(np.int64)).size
    return 1.0 - u / max(1, nodes.size)


def measure(s, k, B, L, n_batches, seed=0):
    g = CSR(s.n_nodes, s.src, s.dst, s.ts)
    nb = (s.n_edges + B - 1) // B
    picks = np.unique(np.linspace(0, nb - 1, min(n_batches, nb)).astype(int))
    res = np.zeros((picks.size, L + 1))
    dts = []
    for r, b in enumerate(picks):
        lo, hi = b * B, min((b + 1) * B, s.n_edges)
        n = np.r_[s.src[lo:hi], s.dst[lo:hi]]
        t = np.r_[s.ts[lo:hi], s.ts[lo:hi]]
        for l in range(L, 0, -1):
            res[r, l] = dup(n, t)
            nn, tj = g.sample(n, t, k)
            if l == L:
                dts.append((t[:, None] - tj).ravel())
            n = np.r_[n, nn.ravel()]
            t = np.r_[t, tj.ravel()]
        res[r, 0] = dup(n)
    dt = np.concatenate(dts)
    return {f"l{l}": float(res[:, l].mean()) for l in range(L + 1)} | {
        "batches": int(picks.size), "dt_lt_1e4_top": float((dt < 10_000).mean()),
        "dt_median_top": float(np.median(dt))}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--batches", type=int, default=200)
    ap.add_argument("--set", nargs="*", default=[])
    ap.add_argument("--json", default=None)
    a = ap.parse_args()
    cfg = get_config(a.config)
    sc = cfg.stream
    over = {}
    for kv in a.set:
        k, v = kv.split("=")
        over[k] = type(getattr(sc, k))(v)
    if over:
        sc = dataclasses.replace(sc, **over)
    s = make_stream(sc, with_features=False)
    r = measure(s, cfg.model.n_neighbors, cfg.model.batch, cfg.model.n_layers, a.batches)
    r["config"] = a.config
    r["stream"] = dataclasses.asdict(sc)
    print(json.dumps(r))
    if a.json:
        json.dump(r, open(a.json, "w"), indent=1)


if __name__ == "__main__":
    main()
