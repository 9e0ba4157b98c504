"""Seeded synthetic CTDG edge streams (SURVEY 8(d) input recipe).

A stream is a list of edges (src_i, dst_i, t_i), i = 0..E-1, with t
non-decreasing; edge id = i + 1 (row 0 of the edge-feature table is
padding). Node ids are 1..V (row 0 of the node-feature table is
padding).

Recipe (shape only, numpy PCG64 seeded):
  * activity is organised in sessions: a session belongs to one user (or one
    source node), starts at a uniform time in [0, max_t] and has a geometric
    number of events separated by Pareto gaps, so the time deltas a
    most-recent sampler sees follow a power law clustered near 0 (Fig. 4,
    P:L168-172);
  * bipartite streams model JODIE's repetitive behaviour: inside a
    session the user repeats its previous item with probability p_rep,
    otherwise it draws an item by Zipf popularity;
  * homogeneous streams draw both endpoints by Zipf popularity, no self-loops;
  * edge and node features are N(0,1) float32 (node features are
    random, not the paper's zero vectors, so node-feature gathers are
    observable in tests).
"""
from dataclasses import dataclass

import numpy as np

from .configs import StreamConfig, CONFIGS


@dataclass
class Stream:
    name: str
    n_nodes: int
    n_edges: int
    src: np.ndarray        # int32 [E]
    dst: np.ndarray        # int32 [E]
    ts: np.ndarray         # uint32 [E], non-decreasing
    node_feat: np.ndarray  # float32 [(V+1) x d_n], row 0 = 0
    edge_feat: np.ndarray  # float32 [(E+1) x d_e], row 0 = 0

    @property
    def d_n(self):
        return self.node_feat.shape[1]

    @property
    def d_e(self):
        return self.edge_feat.shape[1]


def _zipf_weights(n, a, rng):
    w = 1.0 / np.arange(1, n + 1, dtype=np.float64) ** a
    rng.shuffle(w)
    return w / w.sum()


def _session_times(cfg: StreamConfig, rng, n_events):
    """Return (session_id per event, event time) for >= n_events events."""
    n_sess = max(1, int(n_events / cfg.session_mean * 1.3) + 8)
    lens = rng.geometric(1.0 / cfg.session_mean, size=n_sess)
    while lens.sum() < n_events:
        lens = np.concatenate([lens, rng.geometric(1.0 / cfg.session_mean, size=n_sess)])
    total = int(lens.sum())
    sess = np.repeat(np.arange(lens.size), lens)
    starts = rng.integers(0, cfg.max_t + 1, size=lens.size).astype(np.float64)
    # Pareto(alpha=1.2) gaps, scale gap_scale seconds, floored to integer seconds
    gaps = np.floor(cfg.gap_scale * (rng.pareto(1.2, size=total))) + cfg.min_gap
    first = np.r_[0, np.cumsum(lens)[:-1]]
    gaps[first] = 0.0
    # cumulative gap inside each session
    cg = np.cumsum(gaps)
    cg -= np.repeat(cg[first], lens)
    t = np.minimum(starts[sess] + cg, float(cfg.max_t))
    return sess, lens, first, t


def make_stream(cfg, n_edges: int = None, with_features: bool = True) -> Stream:
    """Generate the seeded stream for `cfg` (a StreamConfig or a CONFIGS name).

    n_edges (optional) truncates the stream to its first n_edges events after
    sorting (same seed => a prefix of the full stream's law, used by tests).
    """
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg].stream
    rng = np.random.Generator(np.random.PCG64(cfg.seed))
    E = cfg.n_edges
    V = cfg.n_nodes
    sess, lens, first, t = _session_times(cfg, rng, E)
    total = t.size
    if cfg.bipartite:
        n_users = cfg.n_users
        n_items = V - n_users
        wu = _zipf_weights(n_users, cfg.zipf_user, rng)
        wi = _zipf_weights(n_items, cfg.zipf_item, rng)
        sess_user = rng.choice(n_users, size=lens.size, p=wu) + 1
        src = sess_user[sess]
        item_draw = rng.choice(n_items, size=total, p=wi) + 1 + n_users
        rep = rng.random(total) < cfg.p_rep
        rep[first] = False
        # forward-fill: a repeated event takes the item of the last non-repeat event
        last_nonrep = np.where(~rep, np.arange(total), 0)
        last_nonrep = np.maximum.accumulate(last_nonrep)
        dst = item_draw[last_nonrep]
    else:
        wn = _zipf_weights(V, cfg.zipf_user, rng)
        sess_node = rng.choice(V, size=lens.size, p=wn) + 1
        src = sess_node[sess]
        dst = rng.choice(V, size=total, p=wn) + 1
        clash = dst == src
        while clash.any():
            dst[clash] = rng.choice(V, size=int(clash.sum()), p=wn) + 1
            clash = dst == src
    keep = np.sort(rng.choice(total, size=E, replace=False))
    order = keep[np.argsort(t[keep], kind="stable")]
    src = src[order].astype(np.int32)
    dst = dst[order].astype(np.int32)
    ts = t[order].astype(np.uint32)
    if n_edges is not None:
        src, dst, ts = src[:n_edges], dst[:n_edges], ts[:n_edges]
        E = int(n_edges)
    if with_features:
        frng = np.random.Generator(np.random.PCG64(cfg.seed + 1_000_003))
        node_feat = frng.standard_normal((V + 1, cfg.d_n), dtype=np.float32)
        node_feat[0] = 0.0
        edge_feat = frng.standard_normal((E + 1, cfg.d_e), dtype=np.float32)
        edge_feat[0] = 0.0
    else:
        node_feat = np.zeros((V + 1, cfg.d_n), np.float32)
        edge_feat = np.zeros((1, cfg.d_e), np.float32)
    return Stream(cfg.name, V, E, src, dst, ts, node_feat, edge_feat)


def batches(n_edges: int, batch: int):
    """Chronological batch boundaries [(lo, hi)], the last one partial (R13)."""
    return [(lo, min(lo + batch, n_edges)) for lo in range(0, n_edges, batch)]


def negatives(s: Stream, seed: int = 0) -> np.ndarray:
    """Seeded negative destinations for link-prediction evaluation (NEXT-3, the TGAT protocol
    the paper's task follows): for every edge, a node drawn uniformly from the set of
    destination nodes of the stream. An input of the evaluation, not part of the method."""
    rng = np.random.Generator(np.random.PCG64(1_000_033 + seed))
    pool = np.unique(s.dst)
    return pool[rng.integers(0, pool.size, size=s.n_edges)].astype(np.int32)
