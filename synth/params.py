"""Seeded TGAT model parameters packed in the flat layout include/tg.h documents.

Layout (row-major, PyTorch `Linear` weight = [out x in]); D = d_n + d_e + d_t:
  for l = 1..L:
    W_q[D x D], W_k[D x D], W_v[D x D]        (no bias, [37])
    W_fc[D x D], b_fc[D]
    ln_g[D], ln_b[D]
    W_m1[d_n x (D + d_n)], b_m1[d_n]
    W_m2[d_n x d_n], b_m2[d_n]
  shared:
    omega[d_t], phi[d_t]                       (Eq. 8)
    W_a1[d_n x 2 d_n], b_a1[d_n], W_a2[1 x d_n], b_a2[1]   (affinity MLP, R10)

Init follows the [37]-style scheme of SURVEY 8(d): normal(0, sqrt(2/(D+d_k)))
for W_q/W_k/W_v, Xavier-normal for the fc layers, omega = 1/10^linspace(0,9,d_t),
phi ~ U(-0.5, 0.5) and non-trivial LayerNorm gamma/beta so every parameter is
exercised. Values only; this module computes nothing of the method.
"""
import numpy as np


def param_count(L, d_n, d_e, d_t):
    D = d_n + d_e + d_t
    per_layer = 4 * D * D + D + 2 * D + d_n * (D + d_n) + d_n + d_n * d_n + d_n
    shared = 2 * d_t + d_n * 2 * d_n + d_n + d_n + 1
    return L * per_layer + shared


def make_params(L, H, d_n, d_e, d_t=None, seed=1234) -> np.ndarray:
    d_t = d_n if d_t is None else d_t
    D = d_n + d_e + d_t
    assert D % H == 0, "D must divide into heads"
    d_k = D // H
    rng = np.random.Generator(np.random.PCG64(seed))
    parts = []

    def normal(shape, std):
        parts.append(rng.normal(0.0, std, size=shape).astype(np.float32).ravel())

    def xavier(out_f, in_f):
        normal((out_f, in_f), np.sqrt(2.0 / (in_f + out_f)))

    def uniform(n, bound):
        parts.append(rng.uniform(-bound, bound, size=n).astype(np.float32))

    for _ in range(L):
        for _w in range(3):
            normal((D, D), np.sqrt(2.0 / (D + d_k)))
        xavier(D, D)
        uniform(D, 1.0 / np.sqrt(D))
        parts.append((1.0 + 0.1 * rng.standard_normal(D)).astype(np.float32))
        parts.append((0.1 * rng.standard_normal(D)).astype(np.float32))
        xavier(d_n, D + d_n)
        uniform(d_n, 1.0 / np.sqrt(D + d_n))
        xavier(d_n, d_n)
        uniform(d_n, 1.0 / np.sqrt(d_n))
    parts.append((1.0 / 10 ** np.linspace(0, 9, d_t)).astype(np.float32))
    parts.append(rng.uniform(-0.5, 0.5, size=d_t).astype(np.float32))
    xavier(d_n, 2 * d_n)
    uniform(d_n, 1.0 / np.sqrt(2 * d_n))
    xavier(1, d_n)
    uniform(1, 1.0 / np.sqrt(d_n))
    flat = np.concatenate(parts).astype(np.float32)
    assert flat.size == param_count(L, d_n, d_e, d_t)
    return flat
