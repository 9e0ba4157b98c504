"""ORACLE (test infrastructure only) -- TGOpt Alg. 1 / 2 / 3 followed step by step.

Embed(l, ns, ts) of Alg. 1: DedupFilter (Alg. 2),
ComputeKeys, CacheLookup, NghLookup, recursive
Embed(l-1, ns U ns_ngh, ...) (Alg. 1 l.12), TimeEncode with a precomputed
window, M (Eqs. 6-7), CacheStore (Alg. 3) with the
FIFO memory limit, DedupInvert (Alg. 1 l.20).

Two uses:
  * the invariance pin: with compute=True its embeddings equal the plain
    oracle.tgat forward (the optimisations are semantic-preserving, P:L37,
    P:L176);
  * exact integer counters per batch (unique / hits / misses / evictions /
    time-table hits) that the GPU path must reproduce bit-exactly; with
    compute=False it runs the bookkeeping only (fast).

Readings used: R8 dedup order = first occurrence; R9 cache layers
1..L-1, one table per layer, key = Hash(i, t); R11 FIFO = keep the newest
`limit` stored items; the layer-(l-1) input list is [miss targets ; their
sampled neighbours row-major] (Alg. 1 l.12).
"""
import numpy as np

from .tgat import time_encode


def hash_key(n, t):
    """Hash(n, t): 64-bit key from two 32-bit values by shift and OR (R4)."""
    return (int(n) << 32) | (int(t) & 0xFFFFFFFF)


def dedup_filter(ns, ts):
    """Alg. 2 verbatim: unique (n, t) in first-occurrence order plus inv_idx."""
    ns_u, ts_u, inv = [], [], []
    processed = {}
    for i in range(len(ns)):
        n, t = int(ns[i]), int(ts[i])
        key = hash_key(n, t)
        if key in processed:
            inv.append(processed[key])
        else:
            idx = len(ns_u)
            inv.append(idx)
            ns_u.append(n)
            ts_u.append(t)
            processed[key] = idx
    return np.array(ns_u, np.int64), np.array(ts_u, np.int64), np.array(inv, np.int64)


class FifoCache:
    """Key -> embedding table with a FIFO item limit (Alg. 3; R11).

    Items are kept in insertion order; after a store the table holds the newest
    min(limit, stored) items. A key stored again while present (possible only
    with DedupFilter disabled) keeps its newest copy.
    """

    def __init__(self, limit):
        self.limit = int(limit)
        self.pos = {}         # key -> logical insertion position
        self.vals = {}        # key -> vector
        self.keys = []        # logical position -> key
        self.size = 0

    def head(self):
        return len(self.keys)

    def live(self, key):
        p = self.pos.get(key)
        return p is not None and p >= self.head() - self.size

    def lookup(self, keys):
        """CacheLookup: hit mask and the hit vectors."""
        hits = np.array([self.live(k) for k in keys], bool)
        return hits, [self.vals.get(k) if h else None for k, h in zip(keys, hits)]

    def store(self, keys, H):
        """CacheStore (Alg. 3): evict oldest items beyond the limit, insert in order.

        Returns the number of live items evicted by this call.
        """
        before = self.size
        for i, k in enumerate(keys):
            self.pos[k] = len(self.keys)
            self.keys.append(k)
            if H is not None:
                self.vals[k] = H[i]
        new = before + len(keys)
        self.size = min(new, self.limit)
        evicted_total = new - self.size
        # evicted items that were live before this store (not counting same-call overflow)
        return min(evicted_total, before)


class TGOptSim:
    """Alg. 1 with the three toggles of the ablation: dedup, cache, time table."""

    COUNTERS = ("n", "unique", "lookups", "hits", "misses", "evicted")

    def __init__(self, tgat, cache_limit=2_000_000, time_window=10_000,
                 dedup=True, cache=True, ttable=True, compute=True):
        self.t = tgat
        self.m = tgat.m
        self.g = tgat.g
        self.k = tgat.k
        self.dedup, self.use_cache, self.ttable, self.compute = dedup, cache, ttable, compute
        self.W = int(time_window)
        self.caches = {l: FifoCache(cache_limit) for l in range(1, self.m.L)}
        if self.ttable and compute:
            # precomputed window [0, W), same formula as the direct path
            self.table = time_encode(np.arange(self.W), self.m.omega32, self.m.phi32)
        # TimeEncode(0) computed once ahead of time
        self.phi0 = time_encode(np.zeros(1, np.int64), self.m.omega32, self.m.phi32)[0]
        self.reset_counters()

    def reset_counters(self):
        self.c = {l: dict.fromkeys(self.COUNTERS, 0) for l in range(0, self.m.L + 1)}
        self.t_hits = 0
        self.t_direct = 0

    def time_encode(self, delta):
        """TimeEncode with precomputation: table if dt < W else direct."""
        delta = np.asarray(delta, np.int64)
        inwin = (delta >= 0) & (delta < self.W) if self.ttable else np.zeros(delta.shape, bool)
        self.t_hits += int(inwin.sum())
        self.t_direct += int((~inwin).sum())
        if not self.compute:
            return None
        out = np.empty(delta.shape + (self.m.d_t,))
        out[inwin] = self.table[delta[inwin]] if self.ttable else 0
        out[~inwin] = time_encode(delta[~inwin], self.m.omega32, self.m.phi32)
        return out

    def embed(self, l, ns, ts):
        ns = np.asarray(ns, np.int64)
        ts = np.asarray(ts, np.int64)
        c = self.c[l]
        c["n"] += ns.size
        if l == 0:
            return self.t.X[ns] if self.compute else None               # Alg. 1 l.2-4
        if self.dedup:
            ns, ts, inv = dedup_filter(ns, ts)                          # l.6
        else:
            inv = None
        c["unique"] += ns.size
        keys = [hash_key(n, t) for n, t in zip(ns, ts)]                 # l.7
        cached_layer = self.use_cache and l < self.m.L                  # R9
        if cached_layer:
            hits, hv = self.caches[l].lookup(keys)                      # l.8
            c["lookups"] += len(keys)
        else:
            hits, hv = np.zeros(ns.size, bool), None
        c["hits"] += int(hits.sum())
        H = np.empty((ns.size, self.m.d_n)) if self.compute else None
        if self.compute and hits.any():
            H[hits] = np.stack([v for v in hv if v is not None])
        miss = ~hits
        m = int(miss.sum())
        c["misses"] += m
        if m:                                                            # l.9
            mns, mts = ns[miss], ts[miss]                                # l.10
            nbr, eid, nts = self.g.sample_many(mns, mts, self.k)         # l.11
            Hp = self.embed(l - 1, np.concatenate([mns, nbr.ravel()]),   # l.12
                            np.concatenate([mts, nts.ravel()]))
            ph = self.time_encode(mts[:, None] - nts)                   # l.13-14
            if self.compute:
                hs = Hp[:m]
                hn = Hp[m:].reshape(m, self.k, self.m.d_n)
                Hm = self._M(l, hs, nbr, eid, ph, hn)                    # l.15-16
            else:
                Hm = None
            if cached_layer:
                c["evicted"] += self.caches[l].store([keys[i] for i in np.flatnonzero(miss)], Hm)  # l.17
            if self.compute:
                H[miss] = Hm                                             # l.18
        if self.compute and inv is not None:
            H = H[inv]                                                   # l.20
        return H

    def _M(self, l, hs, nbr, eid, ph, hn):
        from .tgat import attention, merge_ffn
        m = self.m
        n = hs.shape[0]
        q = np.concatenate([hs, np.zeros((n, m.d_e)), np.broadcast_to(self.phi0, (n, m.d_t))], 1)
        ef = self.t.E[eid].astype(np.float64)
        kv = np.concatenate([hn, ef, ph], 2)
        r = attention(m.layers[l - 1], q, kv, nbr == 0, m.H)
        return merge_ffn(m.layers[l - 1], r, hs)

    def infer_batch(self, src, dst, ts):
        src = np.asarray(src, np.int64)
        dst = np.asarray(dst, np.int64)
        ts = np.asarray(ts, np.int64)
        B = src.size
        H = self.embed(self.m.L, np.concatenate([src, dst]), np.concatenate([ts, ts]))
        if not self.compute:
            return None, None
        return H, self.t.score(H[:B], H[B:])

    def counters(self):
        """Flat counter dict: layer-l entries plus time-table hits/direct."""
        out = {}
        for l, d in self.c.items():
            for k, v in d.items():
                out[f"l{l}_{k}"] = v
        out["t_table"] = self.t_hits
        out["t_direct"] = self.t_direct
        return out
