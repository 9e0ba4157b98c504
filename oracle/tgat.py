"""ORACLE (test infrastructure only) -- baseline TGAT forward, float64.

Written from PAPER.md (P:Lnnn = line of /root/reference/PAPER.md) and the
readings R1..R17 of DESIGN.md. No dedup, no memoization, no time table: this
is the plain definition TGOpt's optimisations must preserve (P:L37, P:L176,
P:L384).

Precision: float64 throughout, except the argument of Eq. 8's cosine, which is
formed in float32 exactly as the fp32 model the paper runs ("32-bit
floats"; R5): arg = fl32(fl32((float)dt * omega) + phi), then cos in float64.
"""
import numpy as np


# ----------------------------------------------------------------------------
# Parameters: flat float32 array in the layout of include/tg.h / DESIGN.md.
# (Parsed here independently of the CUDA library.)
# ----------------------------------------------------------------------------
class Model:
    def __init__(self, flat, n_layers, n_heads, d_n, d_e, d_t=None):
        d_t = d_n if d_t is None else d_t
        self.L, self.H, self.d_n, self.d_e, self.d_t = n_layers, n_heads, d_n, d_e, d_t
        D = self.D = d_n + d_e + d_t
        assert D % n_heads == 0
        self.d_k = D // n_heads
        flat = np.asarray(flat, dtype=np.float32)
        off = [0]

        def take(*shape):
            n = int(np.prod(shape))
            a = flat[off[0]:off[0] + n].reshape(shape)
            off[0] += n
            return a

        self.layers = []
        for _ in range(n_layers):
            p = {}
            p["Wq"], p["Wk"], p["Wv"] = take(D, D), take(D, D), take(D, D)
            p["Wfc"], p["bfc"] = take(D, D), take(D)
            p["ln_g"], p["ln_b"] = take(D), take(D)
            p["Wm1"], p["bm1"] = take(d_n, D + d_n), take(d_n)
            p["Wm2"], p["bm2"] = take(d_n, d_n), take(d_n)
            self.layers.append({k: v.astype(np.float64) for k, v in p.items()})
        self.omega32 = take(d_t).copy()       # kept float32: Eq. 8 argument (R5)
        self.phi32 = take(d_t).copy()
        self.Wa1, self.ba1 = take(d_n, 2 * d_n).astype(np.float64), take(d_n).astype(np.float64)
        self.Wa2, self.ba2 = take(1, d_n).astype(np.float64), take(1).astype(np.float64)
        assert off[0] == flat.size, (off[0], flat.size)


# ----------------------------------------------------------------------------
# Temporal graph and most-recent-k sampler (R6, R7, R14)
# ----------------------------------------------------------------------------
class TemporalGraph:
    """Undirected temporal multigraph (graphs are treated as undirected).

    adj[i] holds (j, e, t_e) for every edge e=(i,j) or (j,i); sorted by (t_e, e)
    ascending (R6). Edge ids are 1-based in stream order.
    """

    def __init__(self, n_nodes, src, dst, ts):
        src = np.asarray(src, np.int64)
        dst = np.asarray(dst, np.int64)
        ts = np.asarray(ts, np.int64)
        E = src.size
        eid = np.arange(1, E + 1, dtype=np.int64)
        node = np.concatenate([src, dst])
        nbr = np.concatenate([dst, src])
        ee = np.concatenate([eid, eid])
        tt = np.concatenate([ts, ts])
        order = np.lexsort((ee, tt, node))      # primary: node, then t, then edge id
        self.nbr = nbr[order]
        self.eid = ee[order]
        self.t = tt[order]
        counts = np.bincount(node, minlength=n_nodes + 1)
        self.indptr = np.zeros(n_nodes + 2, np.int64)
        self.indptr[1:] = np.cumsum(counts)
        self.n_nodes = n_nodes

    def sample(self, i, t, k):
        """N(i,t) = {j : e_ij(t_j), t_j < t}, the k most recent.

        Returns k slots right-aligned in ascending (t_j, e) order; leading empty
        slots are (node 0, edge 0, t 0) (R6, R7).
        """
        lo, hi = self.indptr[i], self.indptr[i + 1]
        p = lo + int(np.searchsorted(self.t[lo:hi], t, side="left"))   # strict t_j < t
        a = max(lo, p - k)
        cnt = p - a
        nb = np.zeros(k, np.int64)
        ed = np.zeros(k, np.int64)
        tj = np.zeros(k, np.int64)
        if cnt:
            nb[k - cnt:] = self.nbr[a:p]
            ed[k - cnt:] = self.eid[a:p]
            tj[k - cnt:] = self.t[a:p]
        return nb, ed, tj

    def sample_many(self, nodes, ts, k):
        n = len(nodes)
        nb = np.zeros((n, k), np.int64)
        ed = np.zeros((n, k), np.int64)
        tj = np.zeros((n, k), np.int64)
        for r in range(n):
            nb[r], ed[r], tj[r] = self.sample(int(nodes[r]), int(ts[r]), k)
        return nb, ed, tj


# ----------------------------------------------------------------------------
# Eq. 8 time encoding; Phi(0) = cos(phi)
# ----------------------------------------------------------------------------
def time_encode(delta, omega32, phi32):
    """Phi(dt)[c] = cos(omega_c * dt + phi_c) (Eq. 8).

    dt is an exact integer (R4) converted to float32 round-to-nearest; the mul
    and the add are each rounded to float32 (R5), the cosine is float64.
    """
    d32 = np.asarray(delta, np.int64).astype(np.float32)
    arg = np.multiply(d32[..., None], omega32, dtype=np.float32)
    arg = np.add(arg, phi32, dtype=np.float32)
    return np.cos(arg.astype(np.float64))


# ----------------------------------------------------------------------------
# Attention operator M (Eq. 6, P:L85, P:L91 -> TGAT [37]; reading R1, R3)
# ----------------------------------------------------------------------------
def attention(p, q, kv, mask, n_heads):
    """r = LayerNorm(W_fc . concat_h softmax(Q_h K_h^T / sqrt(d_k)) V_h + b_fc + q).

    q: [n, D] query z_i (Eq. 4); kv: [n, k, D] keys/values z_j (Eq. 5);
    mask: [n, k] True where the slot is padding (score replaced by -1e10, R7).
    Heads are contiguous blocks of d_k = D / H output rows (R1).
    """
    n, k, D = kv.shape
    dk = D // n_heads
    Q = q @ p["Wq"].T                                  # [n, D]
    kv2 = kv.reshape(n * k, D)
    K = (kv2 @ p["Wk"].T).reshape(n, k, D)             # [n, k, D]
    V = (kv2 @ p["Wv"].T).reshape(n, k, D)
    Qh = Q.reshape(n, n_heads, dk)
    Kh = K.reshape(n, k, n_heads, dk)
    Vh = V.reshape(n, k, n_heads, dk)
    s = np.matmul(Qh[:, :, None, :], Kh.transpose(0, 2, 3, 1))[:, :, 0, :] / np.sqrt(dk)  # [n, H, k]
    s = np.where(mask[:, None, :], -1e10, s)
    s = s - s.max(axis=2, keepdims=True)
    a = np.exp(s)
    a = a / a.sum(axis=2, keepdims=True)
    o = np.matmul(a[:, :, None, :], Vh.transpose(0, 2, 1, 3))[:, :, 0, :].reshape(n, D)   # [n, H*dk]
    y = o @ p["Wfc"].T + p["bfc"]
    z = y + q
    mu = z.mean(axis=1, keepdims=True)
    var = ((z - mu) ** 2).mean(axis=1, keepdims=True)     # biased variance, eps 1e-5 (R1)
    return (z - mu) / np.sqrt(var + 1e-5) * p["ln_g"] + p["ln_b"]


def merge_ffn(p, r, hs):
    """Eq. 7: h = W_m2 ReLU(W_m1 [r || h^(l-1)] + b_m1) + b_m2."""
    x = np.concatenate([r, hs], axis=1)
    z = np.maximum(x @ p["Wm1"].T + p["bm1"], 0.0)
    return z @ p["Wm2"].T + p["bm2"]


# ----------------------------------------------------------------------------
# Recursive embedding (Eqs. 4-7) and link score (R10)
# ----------------------------------------------------------------------------
class TGAT:
    def __init__(self, model: Model, graph: TemporalGraph, node_feat, edge_feat, k, chunk=1024):
        self.m, self.g, self.k, self.chunk = model, graph, k, chunk
        self.X = np.asarray(node_feat, np.float64)
        self.E = np.asarray(edge_feat, np.float32)     # converted per gather (memory)

    def layer(self, l, hs, nodes_ts, nbr, eid, nts, hn):
        """One application of Eqs. 4-7 at layer l for targets with gathered inputs."""
        m = self.m
        ts = nodes_ts
        n = hs.shape[0]
        out = np.empty((n, m.d_n))
        phi0 = time_encode(np.zeros(1, np.int64), m.omega32, m.phi32)[0]
        for a in range(0, n, self.chunk):
            b = min(n, a + self.chunk)
            c = b - a
            q = np.concatenate([hs[a:b], np.zeros((c, m.d_e)), np.broadcast_to(phi0, (c, m.d_t))], 1)
            ef = self.E[eid[a:b]].astype(np.float64)
            ph = time_encode(ts[a:b, None] - nts[a:b], m.omega32, m.phi32)
            kv = np.concatenate([hn[a:b], ef, ph], axis=2)
            r = attention(m.layers[l - 1], q, kv, nbr[a:b] == 0, m.H)
            out[a:b] = merge_ffn(m.layers[l - 1], r, hs[a:b])
        return out

    def embed(self, l, nodes, ts):
        """h^(l)(i, t) for each target <i, t> (recursion down to h^(0) = x_i)."""
        nodes = np.asarray(nodes, np.int64)
        ts = np.asarray(ts, np.int64)
        if l == 0:
            return self.X[nodes]
        hs = self.embed(l - 1, nodes, ts)
        nbr, eid, nts = self.g.sample_many(nodes, ts, self.k)
        n = nodes.size
        hn = self.embed(l - 1, nbr.ravel(), nts.ravel()).reshape(n, self.k, self.m.d_n)
        return self.layer(l, hs, ts, nbr, eid, nts, hn)

    def score(self, h_src, h_dst):
        """Affinity MLP + sigmoid on (h_src, h_dst) (R10, TGAT [37])."""
        m = self.m
        x = np.concatenate([h_src, h_dst], axis=1)
        z = np.maximum(x @ m.Wa1.T + m.ba1, 0.0)
        logit = (z @ m.Wa2.T + m.ba2)[:, 0]
        return 1.0 / (1.0 + np.exp(-logit))

    def infer_batch(self, src, dst, ts):
        """One chronological batch: targets src || dst at the edge time."""
        src = np.asarray(src, np.int64)
        dst = np.asarray(dst, np.int64)
        ts = np.asarray(ts, np.int64)
        B = src.size
        H = self.embed(self.m.L, np.concatenate([src, dst]), np.concatenate([ts, ts]))
        return H, self.score(H[:B], H[B:])
