"""Pins for the oracle (CPU only): the oracle is checked against things other
than itself -- the paper's worked examples (tests/golden), closed forms, brute
force on tiny inputs, library routines (torch float64) and invariants.
"""
import json
import math
import os

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from synth import make_stream, make_params, get_config
from oracle.tgat import Model, TemporalGraph, TGAT, time_encode, attention, merge_ffn
from oracle.tgopt import TGOptSim, dedup_filter, hash_key, FifoCache
from tests._bruteforce import BruteTGAT

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _setup(name, **over):
    cfg = get_config(name, **over)
    s = make_stream(name)
    mc = cfg.model
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    m = Model(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    g = TemporalGraph(s.n_nodes, s.src, s.dst, s.ts)
    return cfg, s, flat, m, g, TGAT(m, g, s.node_feat, s.edge_feat, mc.n_neighbors)


# --------------------------------------------------------------------- dedup
def test_fig1_dedup_example():
    gd = json.load(open(os.path.join(GOLD, "fig1_dedup.json")))
    ns, ts, inv = dedup_filter(gd["nodes"], gd["ts"])
    assert ns.tolist() == gd["unique_nodes"]
    assert ts.tolist() == gd["unique_ts"]
    assert inv.tolist() == gd["inv_idx"]


def test_dedup_matches_numpy_unique_first_occurrence():
    rng = np.random.default_rng(0)
    for n in (1, 7, 300, 5000):
        ns = rng.integers(0, 40, n)
        ts = rng.integers(0, 6, n)
        u_n, u_t, inv = dedup_filter(ns, ts)
        pairs = np.stack([ns, ts], 1)
        uniq, first, inverse = np.unique(pairs, axis=0, return_index=True, return_inverse=True)
        order = np.argsort(first)                      # first-occurrence order (Alg. 2)
        assert np.array_equal(np.stack([u_n, u_t], 1), uniq[order])
        rank = np.empty_like(order)
        rank[order] = np.arange(order.size)
        assert np.array_equal(inv, rank[inverse.ravel()])
        assert np.array_equal(u_n[inv], ns) and np.array_equal(u_t[inv], ts)


def test_dedup_empty():
    ns, ts, inv = dedup_filter([], [])
    assert ns.size == 0 and ts.size == 0 and inv.size == 0


def test_hash_key_injective_roundtrip():
    rng = np.random.default_rng(1)
    n = rng.integers(0, 2**31 - 1, 2000)
    t = rng.integers(0, 2**32 - 1, 2000, dtype=np.uint64)
    keys = {hash_key(a, b) for a, b in zip(n, t)}
    assert len(keys) == len(set(zip(n.tolist(), t.tolist())))
    for a, b in zip(n[:50], t[:50]):
        k = hash_key(a, b)
        assert (k >> 32) == int(a) and (k & 0xFFFFFFFF) == int(b)
    assert hash_key(0, 0) == 0 and hash_key(1, 0) == 1 << 32


# ------------------------------------------------------------------- sampler
def test_fig2_sampler_example():
    gd = json.load(open(os.path.join(GOLD, "fig2_sampler.json")))
    names = {v: k for k, v in gd["nodes"].items()}
    e = np.array(gd["edges"])
    k = gd["k"]
    v = gd["nodes"]["v"]
    # the graph before d arrives, and after
    g_before = TemporalGraph(5, e[:3, 0], e[:3, 1], e[:3, 2])
    g_after = TemporalGraph(5, e[:, 0], e[:, 1], e[:, 2])
    t4, t6 = gd["times"]["t4"], gd["times"]["t6"]
    nb, _, _ = g_before.sample(v, t4, k)
    assert [names[int(j)] for j in nb] == gd["expect"]["v@t4"]
    nb6, _, _ = g_after.sample(v, t6, k)
    assert [names[int(j)] for j in nb6] == gd["expect"]["v@t6"]
    nb4b, eid4b, t4b = g_after.sample(v, t4, k)     # purity
    nb4, eid4, tt4 = g_before.sample(v, t4, k)
    assert np.array_equal(nb4, nb4b) and np.array_equal(eid4, eid4b) and np.array_equal(tt4, t4b)


def _brute_sample(src, dst, ts, i, t, k):
    found = []
    for e, (s, d, te) in enumerate(zip(src, dst, ts), start=1):
        if te < t:
            if s == i:
                found.append((te, e, d))
            if d == i:
                found.append((te, e, s))
    found.sort()
    found = found[-k:] if k else []
    pad = k - len(found)
    return ([0] * pad + [x[2] for x in found], [0] * pad + [x[1] for x in found],
            [0] * pad + [x[0] for x in found])


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_sampler_bruteforce(seed):
    rng = np.random.default_rng(seed)
    V, E = 9, 80
    src = rng.integers(1, V + 1, E)
    dst = rng.integers(1, V + 1, E)         # self-loops allowed here (appear twice, R6)
    ts = np.sort(rng.integers(0, 30, E))    # many ties
    g = TemporalGraph(V, src, dst, ts)
    for _ in range(200):
        i = int(rng.integers(0, V + 1))
        t = int(rng.integers(0, 35))
        k = int(rng.integers(0, 6))
        nb, ed, tj = g.sample(i, t, k)
        bn, be, bt = _brute_sample(src, dst, ts, i, t, k)
        assert nb.tolist() == bn and ed.tolist() == be and tj.tolist() == bt
        assert np.all(tj[nb != 0] < t)


# ------------------------------------------------------------- time encoding
def test_time_encode_phi0_is_cos_phi():
    rng = np.random.default_rng(3)
    om = (1.0 / 10 ** np.linspace(0, 9, 17)).astype(np.float32)
    ph = rng.uniform(-3, 3, 17).astype(np.float32)
    out = time_encode(np.zeros(1, np.int64), om, ph)[0]
    assert np.array_equal(out, np.cos(ph.astype(np.float64)))


def test_time_encode_exact_products_closed_form():
    # omega = powers of two and small dt: the fp32 product and sum are exact,
    # so Phi must equal the real cos(omega*dt + phi) (Eq. 8)
    om = np.array([1.0, 0.5, 0.25, 2.0 ** -10, 4.0], np.float32)
    ph = np.array([0.0, 0.25, -0.5, 0.125, 1.0], np.float32)
    dts = np.array([0, 1, 2, 3, 17, 255, 1000], np.int64)
    out = time_encode(dts, om, ph)
    for a, dt in enumerate(dts):
        for c in range(om.size):
            assert out[a, c] == pytest.approx(math.cos(float(om[c]) * dt + float(ph[c])), abs=1e-15)


def test_time_encode_large_dt_rounds_in_fp32():
    # dt > 2^24 is rounded to fp32 first (R4); the product then rounds again (R5)
    om = np.array([1.0], np.float32)
    ph = np.array([0.0], np.float32)
    dt = 2 ** 24 + 1
    out = time_encode(np.array([dt]), om, ph)[0, 0]
    assert out == math.cos(float(2 ** 24))


# ----------------------------------------------------------------- attention
def _rand_attn_inputs(seed, n=5, k=4, dn=6, de=4, H=2):
    rng = np.random.default_rng(seed)
    D = dn + de + dn
    p = {
        "Wq": rng.normal(size=(D, D)), "Wk": rng.normal(size=(D, D)), "Wv": rng.normal(size=(D, D)),
        "Wfc": rng.normal(size=(D, D)) / 4, "bfc": rng.normal(size=D),
        "ln_g": 1 + 0.1 * rng.normal(size=D), "ln_b": 0.1 * rng.normal(size=D),
        "Wm1": rng.normal(size=(dn, D + dn)), "bm1": rng.normal(size=dn),
        "Wm2": rng.normal(size=(dn, dn)), "bm2": rng.normal(size=dn),
    }
    q = rng.normal(size=(n, D))
    kv = rng.normal(size=(n, k, D))
    return p, q, kv, D, H


def test_attention_matches_torch_mha_float64():
    p, q, kv, D, H = _rand_attn_inputs(0)
    n, k = kv.shape[:2]
    mask = np.zeros((n, k), bool)
    mask[1, :2] = True
    mask[3, 0] = True
    r = attention(p, q, kv, mask, H)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a))
    out, _ = F.multi_head_attention_forward(
        t(q)[None], t(kv).transpose(0, 1), t(kv).transpose(0, 1), D, H,
        in_proj_weight=None, in_proj_bias=None, bias_k=None, bias_v=None, add_zero_attn=False,
        dropout_p=0.0, out_proj_weight=t(p["Wfc"]), out_proj_bias=t(p["bfc"]), training=False,
        key_padding_mask=t(mask), need_weights=False, use_separate_proj_weight=True,
        q_proj_weight=t(p["Wq"]), k_proj_weight=t(p["Wk"]), v_proj_weight=t(p["Wv"]))
    ref = F.layer_norm(out[0] + t(q), (D,), t(p["ln_g"]), t(p["ln_b"]), eps=1e-5)
    np.testing.assert_allclose(r, ref.numpy(), rtol=1e-12, atol=1e-12)


def test_attention_k1_closed_form():
    # k = 1: the softmax weight is 1, so r = LN(W_fc W_v kv + b_fc + q)
    p, q, kv, D, H = _rand_attn_inputs(1, k=1)
    r = attention(p, q, kv, np.zeros(kv.shape[:2], bool), H)
    y = kv[:, 0] @ p["Wv"].T @ p["Wfc"].T + p["bfc"] + q
    t = torch.from_numpy
    ref = F.layer_norm(t(y), (D,), t(p["ln_g"]), t(p["ln_b"]), eps=1e-5).numpy()
    np.testing.assert_allclose(r, ref, rtol=1e-12, atol=1e-12)


def test_attention_all_masked_is_uniform():
    # every slot is padding: all scores are -1e10, the weights are uniform 1/k (R7)
    p, q, kv, D, H = _rand_attn_inputs(2)
    n, k = kv.shape[:2]
    r = attention(p, q, kv, np.ones((n, k), bool), H)
    y = kv.mean(axis=1) @ p["Wv"].T @ p["Wfc"].T + p["bfc"] + q
    t = torch.from_numpy
    ref = F.layer_norm(t(y), (D,), t(p["ln_g"]), t(p["ln_b"]), eps=1e-5).numpy()
    np.testing.assert_allclose(r, ref, rtol=1e-11, atol=1e-11)


def test_merge_ffn_matches_torch():
    p, q, kv, D, H = _rand_attn_inputs(3)
    dn = p["Wm2"].shape[0]
    r = np.random.default_rng(4).normal(size=(5, D))
    hs = np.random.default_rng(5).normal(size=(5, dn))
    out = merge_ffn(p, r, hs)
    t = torch.from_numpy
    ref = F.linear(F.relu(F.linear(torch.cat([t(r), t(hs)], 1), t(p["Wm1"]), t(p["bm1"]))),
                   t(p["Wm2"]), t(p["bm2"]))
    np.testing.assert_allclose(out, ref.numpy(), rtol=1e-12, atol=1e-12)


# ----------------------------------------------------------------- recursion
def test_embed_layer0_is_node_features():
    cfg, s, flat, m, g, t = _setup("tiny")
    nodes = np.array([0, 1, 5, 5, 12])
    assert np.array_equal(t.embed(0, nodes, np.zeros(5)), s.node_feat[nodes].astype(np.float64))


@pytest.mark.parametrize("name", ["tiny", "tiny_bip"])
def test_embed_and_score_match_bruteforce(name):
    cfg, s, flat, m, g, t = _setup(name)
    mc = cfg.model
    bf = BruteTGAT(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e, s.src, s.dst, s.ts,
                   s.node_feat, s.edge_feat, mc.n_neighbors)
    lo, hi = s.n_edges - mc.batch, s.n_edges          # last batch: richest neighbourhoods
    H, p = t.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
    B = hi - lo
    for r in range(B):
        hs = bf.embed(mc.n_layers, int(s.src[lo + r]), int(s.ts[lo + r]))
        hd = bf.embed(mc.n_layers, int(s.dst[lo + r]), int(s.ts[lo + r]))
        np.testing.assert_allclose(H[r], hs, rtol=1e-10, atol=1e-10)
        np.testing.assert_allclose(H[B + r], hd, rtol=1e-10, atol=1e-10)
        assert p[r] == pytest.approx(bf.score(hs, hd), rel=1e-10, abs=1e-12)


def test_score_matches_torch():
    cfg, s, flat, m, g, t = _setup("tiny")
    rng = np.random.default_rng(6)
    hs, hd = rng.normal(size=(7, s.d_n)), rng.normal(size=(7, s.d_n))
    tt = torch.from_numpy
    ref = torch.sigmoid(F.linear(F.relu(F.linear(torch.cat([tt(hs), tt(hd)], 1), tt(m.Wa1), tt(m.ba1))),
                                 tt(m.Wa2), tt(m.ba2)))[:, 0]
    np.testing.assert_allclose(t.score(hs, hd), ref.numpy(), rtol=1e-12)


# ----------------------------------------------------- Alg. 1 invariance / counters
@pytest.mark.parametrize("opts", [(True, True, True), (False, True, True), (True, False, True),
                                  (True, True, False), (False, False, False)])
@pytest.mark.parametrize("limit", [2_000_000, 25])
def test_alg1_sim_equals_plain_oracle(opts, limit):
    cfg, s, flat, m, g, t = _setup("tiny_bip")
    mc = cfg.model
    sim = TGOptSim(t, cache_limit=limit, time_window=mc.time_window,
                   dedup=opts[0], cache=opts[1], ttable=opts[2])
    for lo in range(0, s.n_edges, mc.batch):
        hi = min(lo + mc.batch, s.n_edges)
        H0, p0 = t.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        H1, p1 = sim.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        np.testing.assert_allclose(H1, H0, rtol=1e-12, atol=1e-12)
        np.testing.assert_allclose(p1, p0, rtol=1e-12, atol=1e-12)


def test_alg1_sim_bookkeeping_matches_compute_mode():
    cfg, s, flat, m, g, t = _setup("tiny_bip")
    mc = cfg.model
    a = TGOptSim(t, cache_limit=30, time_window=mc.time_window)
    b = TGOptSim(t, cache_limit=30, time_window=mc.time_window, compute=False)
    for lo in range(0, s.n_edges, mc.batch):
        hi = min(lo + mc.batch, s.n_edges)
        a.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        b.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
    assert a.counters() == b.counters()
    assert a.counters()["l1_evicted"] > 0


def test_counters_key_universe_no_eviction():
    # with an unbounded cache every distinct layer-1 key misses exactly once
    # (the key-universe argument behind P:L448's stored-item counts)
    cfg, s, flat, m, g, t = _setup("config1")
    mc = cfg.model
    sim = TGOptSim(t, cache_limit=10**9, time_window=mc.time_window, compute=False)
    keys = set()
    n_batches = 12
    for b in range(n_batches):
        lo, hi = b * mc.batch, (b + 1) * mc.batch
        sim.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        # layer-1 input for L=2: [U_2 ; N(U_2)] (Alg. 1 l.12), recomputed here independently
        ns = np.r_[s.src[lo:hi], s.dst[lo:hi]]
        ts = np.r_[s.ts[lo:hi], s.ts[lo:hi]]
        u = sorted(set(zip(ns.tolist(), ts.tolist())))
        for (i, tt) in u:
            keys.add((i, tt))
            nb, _, tj = g.sample(i, tt, mc.n_neighbors)
            keys.update(zip(nb.tolist(), tj.tolist()))
    c = sim.counters()
    assert c["l1_misses"] == len(keys)
    assert c["l1_hits"] == c["l1_lookups"] - c["l1_misses"]
    assert c["l1_evicted"] == 0
    assert c["l2_unique"] == c["l2_misses"]
    assert c["l0_n"] == c["l1_misses"] * (mc.n_neighbors + 1)


def test_fifo_cache_semantics():
    c = FifoCache(3)
    assert c.store([1, 2], None) == 0
    assert c.store([3, 4], None) == 1          # 1 evicted (oldest first)
    assert [c.live(k) for k in (1, 2, 3, 4)] == [False, True, True, True]
    assert c.store([5, 6, 7, 8], None) == 3    # n > limit: the newest `limit` survive (R11)
    assert [c.live(k) for k in (4, 5, 6, 7, 8)] == [False, False, True, True, True]


# ------------------------------------------------ TimeEncode window counters (Sec. 4.3)
def _brute_deltas(bt, l, i, t, out):
    """Every dt = t - t_j that computing h(l, i, t) encodes, by literal recursion over the
    edge-scan sampler of tests/_bruteforce.py (no dedup, no memo: the baseline of P:L140)."""
    if l == 0:
        return
    _brute_deltas(bt, l - 1, i, t, out)
    for (j, e, tj) in bt.neighbours(i, t):
        out.append(t - tj)                  # padding slot: t_j = 0, dt = t (R7)
        _brute_deltas(bt, l - 1, j, tj, out)


def _window_setup():
    cfg, s, flat, m, g, t = _setup("tiny_bip")
    mc = cfg.model
    bt = BruteTGAT(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e, s.src, s.dst, s.ts,
                   s.node_feat, s.edge_feat, mc.n_neighbors)
    return cfg, s, t, bt


def test_time_table_counter_baseline_matches_bruteforce_window():
    """Phi(dt) comes from the precomputed window iff 0 <= dt < W. With dedup and cache
    off every target of the (k+1)^L expansion is computed, so the per-batch table/direct counts
    are the brute-force count of dt < W over the expansion. W is set to a dt that occurs, so an
    off-by-one (dt <= W) changes the count."""
    cfg, s, t, bt = _window_setup()
    mc = cfg.model
    nb = 4
    deltas = []
    per_batch = []
    for b in range(nb):
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        d = []
        for (i, tt) in list(zip(s.src[lo:hi], s.ts[lo:hi])) + list(zip(s.dst[lo:hi], s.ts[lo:hi])):
            _brute_deltas(bt, mc.n_layers, int(i), int(tt), d)
        per_batch.append(d)
        deltas += d
    pos = sorted(x for x in deltas if x > 0)
    W = pos[len(pos) // 2]
    assert sum(1 for x in deltas if x == W) > 0
    for win in (W, W + 1):
        sim = TGOptSim(t, time_window=win, dedup=False, cache=False, ttable=True, compute=False)
        for b in range(nb):
            lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
            sim.reset_counters()
            sim.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
            c = sim.counters()
            want_tab = sum(1 for x in per_batch[b] if 0 <= x < win)
            assert c["t_table"] == want_tab, (win, b)
            assert c["t_direct"] == len(per_batch[b]) - want_tab
    # table off: everything direct
    sim = TGOptSim(t, time_window=W, dedup=False, cache=False, ttable=False, compute=False)
    sim.infer_batch(s.src[:mc.batch], s.dst[:mc.batch], s.ts[:mc.batch])
    assert sim.counters()["t_table"] == 0 and sim.counters()["t_direct"] == len(per_batch[0])


def test_time_table_counter_with_memo_matches_key_universe():
    """With dedup and an unbounded cache (L = 2), a layer-2 target is computed once per batch
    per distinct (i, t) and a layer-1 key once per stream (the key-universe argument), so
    the stream's table count is the brute-force dt < W count over exactly those targets."""
    cfg, s, t, bt = _window_setup()
    mc = cfg.model
    assert mc.n_layers == 2
    W = mc.time_window
    k = mc.n_neighbors
    sim = TGOptSim(t, cache_limit=10**9, time_window=W, compute=False)
    seen1 = set()
    want_tab = want_all = 0

    def count(i, tt):
        nonlocal want_tab, want_all
        for (j, e, tj) in bt.neighbours(i, tt):
            want_all += 1
            want_tab += 1 if 0 <= tt - tj < W else 0

    for lo in range(0, s.n_edges, mc.batch):
        hi = min(lo + mc.batch, s.n_edges)
        sim.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        top = []
        for (i, tt) in list(zip(s.src[lo:hi], s.ts[lo:hi])) + list(zip(s.dst[lo:hi], s.ts[lo:hi])):
            if (int(i), int(tt)) not in top:
                top.append((int(i), int(tt)))
        for (i, tt) in top:                      # layer 2: every distinct target of the batch
            count(i, tt)
        for (i, tt) in top:                      # layer 1: keys never computed before
            for key in [(i, tt)] + [(j, tj) for (j, e, tj) in bt.neighbours(i, tt)]:
                if key not in seen1:
                    seen1.add(key)
                    count(*key)
    c = sim.counters()
    assert c["l1_misses"] == len(seen1)
    assert c["t_table"] == want_tab and c["t_direct"] == want_all - want_tab
    assert 0 < want_tab < want_all
