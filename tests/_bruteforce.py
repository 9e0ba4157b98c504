"""Pure-Python brute-force TGAT embedding for tiny inputs (a pin for the oracle).

Independent of oracle/: per-target literal recursion (the (k+1)^L expansion of
P:L140), neighbourhoods found by scanning the whole edge list, and the
attention written out with explicit loops over heads, rows and neighbours
(Eq. 6 per TGAT [37], reading R1). Only float32 rounding of Eq. 8's argument
is shared by construction (R5).
"""
import math

import numpy as np


class BruteTGAT:
    def __init__(self, flat, L, H, d_n, d_e, src, dst, ts, X, E, k):
        self.L, self.H, self.dn, self.de, self.dt = L, H, d_n, d_e, d_n
        self.D = d_n + d_e + d_n
        self.k = k
        self.edges = [(int(s), int(d), int(t), i + 1) for i, (s, d, t) in enumerate(zip(src, dst, ts))]
        self.X = [[float(v) for v in row] for row in X]
        self.E = [[float(v) for v in row] for row in E]
        f = [float(v) for v in flat]
        self.f32 = np.asarray(flat, np.float32)
        pos = 0
        D, dn = self.D, d_n

        def mat(r, c):
            nonlocal pos
            m = [f[pos + i * c: pos + (i + 1) * c] for i in range(r)]
            pos += r * c
            return m

        def vec(n):
            nonlocal pos
            v = f[pos:pos + n]
            pos += n
            return v

        self.layers = []
        for _ in range(L):
            Wq, Wk, Wv = mat(D, D), mat(D, D), mat(D, D)
            Wfc, bfc = mat(D, D), vec(D)
            g, b = vec(D), vec(D)
            W1, b1 = mat(dn, D + dn), vec(dn)
            W2, b2 = mat(dn, dn), vec(dn)
            self.layers.append((Wq, Wk, Wv, Wfc, bfc, g, b, W1, b1, W2, b2))
        self.om_pos = pos
        self.omega = self.f32[pos:pos + dn]
        self.phi = self.f32[pos + dn:pos + 2 * dn]
        pos += 2 * dn
        self.Wa1, self.ba1 = mat(dn, 2 * dn), vec(dn)
        self.Wa2, self.ba2 = mat(1, dn), vec(1)

    def neighbours(self, i, t):
        found = []
        for (s, d, te, e) in self.edges:
            if te < t:
                if s == i:
                    found.append((te, e, d))
                if d == i:
                    found.append((te, e, s))
        found.sort()
        found = found[-self.k:] if self.k else []
        pad = [(0, 0, 0)] * (self.k - len(found))
        return [(0, 0, 0) for _ in pad] + [(d, e, te) for (te, e, d) in found]

    def phi_vec(self, dt):
        out = []
        for c in range(self.dt):
            a = np.float32(np.float32(dt) * self.omega[c])
            a = np.float32(a + self.phi[c])
            out.append(math.cos(float(a)))
        return out

    @staticmethod
    def matvec(W, x):
        return [sum(w * v for w, v in zip(row, x)) for row in W]

    def embed(self, l, i, t):
        if l == 0:
            return list(self.X[i])
        Wq, Wk, Wv, Wfc, bfc, g, b, W1, b1, W2, b2 = self.layers[l - 1]
        hs = self.embed(l - 1, i, t)
        q = hs + [0.0] * self.de + self.phi_vec(0)
        slots = self.neighbours(i, t)
        kvs, masks = [], []
        for (j, e, tj) in slots:
            hn = self.embed(l - 1, j, tj)
            kvs.append(hn + list(self.E[e]) + self.phi_vec(t - tj))
            masks.append(j == 0)
        dk = self.D // self.H
        o = []
        Q = self.matvec(Wq, q)
        Ks = [self.matvec(Wk, kv) for kv in kvs]
        Vs = [self.matvec(Wv, kv) for kv in kvs]
        for h in range(self.H):
            sl = slice(h * dk, (h + 1) * dk)
            sc = []
            for m in range(self.k):
                s = sum(a * c for a, c in zip(Q[sl], Ks[m][sl])) / math.sqrt(dk)
                sc.append(-1e10 if masks[m] else s)
            mx = max(sc)
            ex = [math.exp(s - mx) for s in sc]
            z = sum(ex)
            a = [e / z for e in ex]
            for d in range(dk):
                o.append(sum(a[m] * Vs[m][h * dk + d] for m in range(self.k)))
        y = [v + bb + qq for v, bb, qq in zip(self.matvec(Wfc, o), bfc, q)]
        mu = sum(y) / len(y)
        var = sum((v - mu) ** 2 for v in y) / len(y)
        r = [(v - mu) / math.sqrt(var + 1e-5) * gg + bb for v, gg, bb in zip(y, g, b)]
        x = r + hs
        z1 = [max(0.0, v + bb) for v, bb in zip(self.matvec(W1, x), b1)]
        return [v + bb for v, bb in zip(self.matvec(W2, z1), b2)]

    def score(self, hs, hd):
        x = hs + hd
        z = [max(0.0, v + bb) for v, bb in zip(self.matvec(self.Wa1, x), self.ba1)]
        logit = self.matvec(self.Wa2, z)[0] + self.ba2[0]
        return 1.0 / (1.0 + math.exp(-logit))
