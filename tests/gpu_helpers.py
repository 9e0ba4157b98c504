"""Shared helpers of the GPU parity tests (seeded inputs -> library + oracle)."""
import numpy as np

from synth import make_stream, make_params, get_config


def close(a, b, rtol=1e-4, atol=1e-5):
    """Elementwise |a - b| <= atol + rtol |b| (north_star tolerance, R17)."""
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    err = np.abs(a - b)
    bound = atol + rtol * np.abs(b)
    bad = err > bound
    return (not bad.any()), float(err.max(initial=0.0)), int(bad.sum())


def setup(name, n_edges=None, **model_over):
    cfg = get_config(name, **model_over)
    s = make_stream(name, n_edges=n_edges)
    mc = cfg.model
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    return cfg, s, flat


def make_ctx(s, flat, mc, precision=0, opts=7, cache_limit=None, max_targets=None, device=0, superbatch=0):
    from paper_conf_ppopp_wangm23_b200 import Context
    ctx = Context.from_stream(s, device=device)
    ctx.load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                   max_batch_targets=max_targets or 2 * mc.batch,
                   cache_limit=mc.cache_limit if cache_limit is None else cache_limit,
                   time_window=mc.time_window, opts=opts, precision=precision, superbatch=superbatch)
    return ctx


def make_oracle(s, flat, mc):
    from oracle.tgat import Model, TemporalGraph, TGAT
    m = Model(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    g = TemporalGraph(s.n_nodes, s.src, s.dst, s.ts)
    return TGAT(m, g, s.node_feat, s.edge_feat, mc.n_neighbors)
