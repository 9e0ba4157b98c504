"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

Each whole stream (configs[1..4]) runs through ``tg_score_stream`` exactly as ``bench.py``
launches it (default superbatch S, the bench's precision), cold cache. The plain oracle
(oracle/tgat.py) then recomputes a stratified sample of batches one by one -- valid because every
batch's scores are a pure function of (graph, weights, batch) -- and the
per-batch counters of the whole stream are compared bit-exactly with the Alg. 1/3 bookkeeping
simulator (oracle/tgopt.py, compute=False), FIFO eviction included where the stream's key
universe exceeds the 2M-item limit (LastFM: 2E+1 = 2.59M keys).

Tolerances (north_star, R17, R22): fp32-level modes |d| <= 1e-5 + 1e-4|ref| for embeddings and
scores; bf16 GEMM operands rtol 2e-2 with atol 1e-5 for scores and atol 2e-2 for embedding
elements (R22, measured by tools/parity_errors.py).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from tests.gpu_helpers import close, setup, make_ctx, make_oracle

pytestmark = pytest.mark.gpu
TOL = {1: (1e-4, 1e-5), 2: (2e-2, 1e-5), 4: (1e-4, 1e-5)}        # scores: tf32x3 / bf16 / f16x3
EMB_TOL = {1: (1e-4, 1e-5), 2: (2e-2, 2e-2), 4: (1e-4, 1e-5)}    # embedding elements (R22)
BENCH_S = 0                                # bench.py's superbatch: the library default (largest fitting)


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_wangm23_b200 import lib
    lib()


def _run(ctx, s, batch, E=None):
    from paper_conf_ppopp_wangm23_b200 import TG_NCOUNTERS
    E = s.n_edges if E is None else E
    nb = (E + batch - 1) // batch
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    scores = torch.full((E,), -1.0, dtype=torch.float32, device="cuda")
    log = torch.zeros(nb * TG_NCOUNTERS, dtype=torch.int64, device="cuda")
    ctx.score_stream(d(s.src[:E]), d(s.dst[:E]), d(s.ts[:E].view(np.int32)), batch, scores, log)
    torch.cuda.synchronize()
    return scores.cpu().numpy(), log.cpu().numpy().reshape(nb, TG_NCOUNTERS)


def _picks(nb, extra=()):
    """Stratified batch sample: first, second, evenly spaced interior, last (R13 partial)."""
    return sorted(set([0, 1, nb // 4, nb // 2, (3 * nb) // 4, nb - 1] + list(extra)))


def _check_scores(s, flat, mc, scores, picks, prec):
    o = make_oracle(s, flat, mc)
    for b in picks:
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        _, ref = o.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        ok, err, nbad = close(scores[lo:hi], ref, *TOL[prec])
        assert ok, (b, err, nbad)


def _check_counters(s, flat, mc, log, limit):
    from oracle.tgopt import TGOptSim
    from paper_conf_ppopp_wangm23_b200 import counters_dict
    sim = TGOptSim(make_oracle(s, flat, mc), cache_limit=limit, time_window=mc.time_window,
                   compute=False)
    for b, lo in enumerate(range(0, s.n_edges, mc.batch)):
        hi = min(lo + mc.batch, s.n_edges)
        sim.reset_counters()
        sim.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        want = sim.counters()
        got = counters_dict(log[b], mc.n_layers)
        assert got == want, (b, {k: (got[k], want[k]) for k in want if got[k] != want[k]})
    return sim


@pytest.mark.parametrize("name", ["reddit", "wiki", "mooc"])
def test_fullsize_stream_bench_config(name):
    """Whole stream, bench launch config (bf16, default S): sampled scores vs the plain oracle and
    every batch's counters vs the Alg. 1/3 simulator, bit-exact."""
    cfg, s, flat = setup(name)
    mc = cfg.model
    ctx = make_ctx(s, flat, mc, precision=2, superbatch=BENCH_S)
    scores, log = _run(ctx, s, mc.batch)
    assert np.isfinite(scores).all() and (scores >= 0).all() and (scores <= 1).all()
    nb = log.shape[0]
    _check_scores(s, flat, mc, scores, _picks(nb), 2)
    _check_counters(s, flat, mc, log, mc.cache_limit)
    from paper_conf_ppopp_wangm23_b200 import counters_dict
    assert ctx.counters()["l1_misses"] == sum(counters_dict(r, mc.n_layers)["l1_misses"] for r in log)
    ctx.close()


def test_fullsize_reddit_fp32_level():
    """Reddit stream in the fp32-level tensor-core mode (3xTF32): sampled scores at 1e-4/1e-5."""
    cfg, s, flat = setup("reddit")
    mc = cfg.model
    ctx = make_ctx(s, flat, mc, precision=1, superbatch=BENCH_S)
    scores, _ = _run(ctx, s, mc.batch)
    _check_scores(s, flat, mc, scores, _picks(scores.size // mc.batch + 1), 1)
    ctx.close()


def test_fullsize_lastfm_fifo_eviction():
    """LastFM-shaped stream (1.29M edges): 2E+1 > the 2M limit, so FIFO eviction happens inside
    the pass (Alg. 3 l.1-4, R11). Counters (evictions included) bit-exact for every batch;
    sampled scores after the first eviction vs the plain oracle."""
    cfg, s, flat = setup("lastfm")
    mc = cfg.model
    ctx = make_ctx(s, flat, mc, precision=2, superbatch=BENCH_S)
    scores, log = _run(ctx, s, mc.batch)
    _check_counters(s, flat, mc, log, mc.cache_limit)
    from paper_conf_ppopp_wangm23_b200 import counters_dict
    ev = np.array([counters_dict(r, mc.n_layers)["l1_evicted"] for r in log])
    assert ev.sum() > 0, "stream should exercise FIFO eviction"
    first = int(np.argmax(ev > 0))
    nb = log.shape[0]
    _check_scores(s, flat, mc, scores, _picks(nb, [first, first + 1, (first + nb) // 2]), 2)
    ctx.close()


def test_fullsize_large_batch2000():
    """configs[4] shape (1M nodes, 10M edges, batch 2,000), one rank's share of the 8-way split:
    the first 1/8 of the stream, cold cache; sampled batches vs the plain oracle."""
    cfg, s, flat = setup("large")
    mc = cfg.model
    E8 = (s.n_edges // 8 // mc.batch) * mc.batch
    ctx = make_ctx(s, flat, mc, precision=2, superbatch=BENCH_S, max_targets=2 * mc.batch)
    scores, log = _run(ctx, s, mc.batch, E8)       # the graph holds the whole stream (R14)
    nb = log.shape[0]
    _check_scores(s, flat, mc, scores, [0, nb // 2, nb - 1], 2)
    ctx.close()


def test_fullsize_next4_reddit_L3_k8():
    """NEXT-4: the deeper / narrower model, L = 3, k = 8, two cached
    layers (R9) with one index each, on the whole Reddit-shaped stream in bf16 (S is lowered
    to fit the cache passes): every batch's counters bit-exact against the Alg. 1/3
    simulator, sampled scores vs the plain oracle."""
    cfg, s, flat = setup("reddit", n_layers=3, n_neighbors=8)
    mc = cfg.model
    ctx = make_ctx(s, flat, mc, precision=2, superbatch=BENCH_S)
    scores, log = _run(ctx, s, mc.batch)
    _check_counters(s, flat, mc, log, mc.cache_limit)
    nb = log.shape[0]
    _check_scores(s, flat, mc, scores, [0, nb // 2, nb - 1], 2)
    ctx.close()


@pytest.mark.parametrize("prec", [1, 2, 4])
def test_fullsize_embed_parity_bench_config(prec):
    """Element-wise embedding parity in the bench's launch configuration (Reddit shape, k = 20,
    D = 516, default S): the whole stream first runs through tg_score_stream (cold cache, bench
    config), so the layer-1 embeddings of the memo cache were computed by the bench's kernels
    (k_attn_g at D = 516, k = 20); then tg_embed_batch on the src || dst targets of stratified
    batches (layer-1 rows served from the cache, layer 2 computed) is compared with the plain
    oracle's Embed(L) element by element (P:L384 tolerance; R17 / R22)."""
    cfg, s, flat = setup("reddit")
    mc = cfg.model
    ctx = make_ctx(s, flat, mc, precision=prec, superbatch=BENCH_S)
    assert ctx.superbatch() > 1
    scores, log = _run(ctx, s, mc.batch)
    o = make_oracle(s, flat, mc)
    nb = log.shape[0]
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    worst = 0.0
    for b in _picks(nb):
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        nodes = np.r_[s.src[lo:hi], s.dst[lo:hi]].astype(np.int32)
        ts = np.r_[s.ts[lo:hi], s.ts[lo:hi]].astype(np.uint32)
        out = torch.zeros(nodes.size * s.d_n, dtype=torch.float32, device="cuda")
        ctx.embed_batch(d(nodes), d(ts.view(np.int32)), out)
        torch.cuda.synchronize()
        got = out.cpu().numpy().reshape(nodes.size, s.d_n)
        ref, _ = o.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        ok, err, nbad = close(got, ref, *EMB_TOL[prec])
        worst = max(worst, err)
        assert ok, (b, err, nbad)
    c = ctx.counters()
    assert c["l1_misses"] >= 0
    print(f"prec {prec}: max |embedding - oracle| = {worst:.3e} over {len(_picks(nb))} batches")
    ctx.close()


@pytest.mark.parametrize("name,world,prec", [("config1", 2, 1), ("config1", 3, 2), ("wiki", 2, 1)])
def test_batch_range_shards_equal_single_context(name, world, prec):
    """North_star's multi-GPU partition on one GPU: the stream is cut into `world`
    contiguous batch ranges (shard.shard_batches), each processed by its own libtg context with
    its own cold cache, in sequence. The concatenated scores are bit-equal to one context's pass
    over the whole stream (embeddings are pure functions of (i, t), and every kernel is
    row-batch invariant), and each shard's per-batch counters equal the Alg. 1/3 simulator run
    cold on that shard (so the all-reduced totals are their sum)."""
    from paper_conf_ppopp_wangm23_b200.shard import shard_batches
    from paper_conf_ppopp_wangm23_b200 import counters_dict
    from oracle.tgopt import TGOptSim
    cfg, s, flat = setup(name)
    mc = cfg.model
    whole = make_ctx(s, flat, mc, precision=prec)
    ref, _ = _run(whole, s, mc.batch)
    whole.close()
    parts, tot = [], None
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    from paper_conf_ppopp_wangm23_b200 import TG_NCOUNTERS
    for r in range(world):
        b0, b1, e0, e1 = shard_batches(s.n_edges, mc.batch, r, world)
        ctx = make_ctx(s, flat, mc, precision=prec)           # replica of the whole graph (R14)
        sc = torch.full((e1 - e0,), -1.0, dtype=torch.float32, device="cuda")
        log = torch.zeros((b1 - b0) * TG_NCOUNTERS, dtype=torch.int64, device="cuda")
        ctx.score_stream(d(s.src[e0:e1]), d(s.dst[e0:e1]), d(s.ts[e0:e1].view(np.int32)), mc.batch, sc, log)
        torch.cuda.synchronize()
        parts.append(sc.cpu().numpy())
        log = log.cpu().numpy().reshape(b1 - b0, TG_NCOUNTERS)
        sim = TGOptSim(make_oracle(s, flat, mc), cache_limit=mc.cache_limit, time_window=mc.time_window,
                       compute=False)
        for j, lo in enumerate(range(e0, e1, mc.batch)):
            hi = min(lo + mc.batch, e1)
            sim.reset_counters()
            sim.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
            assert counters_dict(log[j], mc.n_layers) == sim.counters(), (r, j)
        raw = ctx.counters_raw()
        tot = raw if tot is None else tot + raw
        ctx.close()
    assert np.array_equal(np.concatenate(parts), ref)
    assert tot is not None and tot.sum() > 0


def _run_neg(ctx, s, neg, batch, E=None):
    from paper_conf_ppopp_wangm23_b200 import TG_NCOUNTERS
    E = s.n_edges if E is None else E
    nb = (E + batch - 1) // batch
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    scores = torch.full((2 * E,), -1.0, dtype=torch.float32, device="cuda")
    log = torch.zeros(nb * TG_NCOUNTERS, dtype=torch.int64, device="cuda")
    ctx.score_stream_neg(d(s.src[:E]), d(s.dst[:E]), d(s.ts[:E].view(np.int32)), d(neg[:E]), batch, scores, log)
    torch.cuda.synchronize()
    sc = scores.cpu().numpy()
    return sc[:E], sc[E:], log.cpu().numpy().reshape(nb, TG_NCOUNTERS)


def _oracle_neg(o, s, neg, lo, hi):
    B = hi - lo
    t = s.ts[lo:hi]
    H = o.embed(o.m.L, np.r_[s.src[lo:hi], s.dst[lo:hi], neg[lo:hi]], np.r_[t, t, t])
    return o.score(H[:B], H[B:2 * B]), o.score(H[:B], H[2 * B:])


@pytest.mark.parametrize("name,prec,E", [("config1", 1, None), ("config1", 2, None), ("reddit", 1, None)])
def test_stream_negatives_parity_ap_auc(name, prec, E):
    """NEXT-3 (TGAT [37]): link prediction with seeded negatives through the superbatched
    stream path (tg_score_stream_neg): every batch's target list is src || dst || neg (3B targets,
    one dedup). Positive and negative scores of stratified batches match the plain oracle (R17 /
    R22), every batch's counters equal the Alg. 1/3 simulator fed the same 3B targets, scores are
    bit-identical at S = 1 and the default S, and AP / AUC over the sampled batches equal the
    oracle's (the random-weight model ranks near chance: this pins the evaluation path, not a
    trained model)."""
    from sklearn.metrics import average_precision_score, roc_auc_score
    from synth import negatives
    from oracle.tgopt import TGOptSim
    from paper_conf_ppopp_wangm23_b200 import counters_dict
    cfg, s, flat = setup(name)
    mc = cfg.model
    neg = negatives(s, seed=1)
    ctx = make_ctx(s, flat, mc, precision=prec, max_targets=3 * mc.batch)
    pos, ngs, log = _run_neg(ctx, s, neg, mc.batch)
    assert ctx.superbatch() > 1
    ctx.close()
    o = make_oracle(s, flat, mc)
    nb = log.shape[0]
    picks = _picks(nb)
    gp, gn, rp, rn = [], [], [], []
    for b in picks:
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        p_ref, n_ref = _oracle_neg(o, s, neg, lo, hi)
        for got, ref in ((pos[lo:hi], p_ref), (ngs[lo:hi], n_ref)):
            ok, err, nbad = close(got, ref, *TOL[prec])
            assert ok, (b, err, nbad)
        gp.append(pos[lo:hi]); gn.append(ngs[lo:hi]); rp.append(p_ref); rn.append(n_ref)
    y = np.r_[np.ones(sum(map(len, gp))), np.zeros(sum(map(len, gn)))]
    g_all, r_all = np.r_[np.concatenate(gp), np.concatenate(gn)], np.r_[np.concatenate(rp), np.concatenate(rn)]
    assert abs(average_precision_score(y, g_all) - average_precision_score(y, r_all)) <= 2e-3
    assert abs(roc_auc_score(y, g_all) - roc_auc_score(y, r_all)) <= 2e-3
    sim = TGOptSim(o, cache_limit=mc.cache_limit, time_window=mc.time_window, compute=False)
    check = range(nb) if name == "config1" else range(0, nb, max(1, nb // 200))
    for b in range(nb):
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        t = s.ts[lo:hi]
        sim.reset_counters()
        sim.embed(mc.n_layers, np.r_[s.src[lo:hi], s.dst[lo:hi], neg[lo:hi]], np.r_[t, t, t])
        if b in check:
            assert counters_dict(log[b], mc.n_layers) == sim.counters(), b
    if name == "config1":
        one = make_ctx(s, flat, mc, precision=prec, max_targets=3 * mc.batch, superbatch=1)
        pos1, ngs1, _ = _run_neg(one, s, neg, mc.batch)
        one.close()
        assert np.array_equal(pos1, pos) and np.array_equal(ngs1, ngs)
