"""Attention-stage experiment: one Reddit-shaped pass, per-stage device times.

    python tools/attn_exp.py [--config reddit] [--window W] [--edges N] [--precision bf16]
Prints attn ms, launches, targets (computed embeddings) and ns per target.
"""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import make_stream, make_params, get_config  # noqa: E402
from paper_conf_ppopp_wangm23_b200 import Context, TG_PREC_BF16, TG_PREC_TF32X3, TG_PREC_FP32  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="reddit")
ap.add_argument("--window", type=int, default=None)
ap.add_argument("--edges", type=int, default=None)
ap.add_argument("--precision", default="bf16")
a = ap.parse_args()
cfg = get_config(a.config)
mc = cfg.model
s = make_stream(a.config, n_edges=a.edges)
flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
prec = {"bf16": TG_PREC_BF16, "tf32x3": TG_PREC_TF32X3, "fp32": TG_PREC_FP32}[a.precision]
W = a.window if a.window is not None else mc.time_window
ctx = Context.from_stream(s).load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                                        max_batch_targets=2 * mc.batch, cache_limit=mc.cache_limit,
                                        time_window=W, precision=prec)
dev = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
src, dst, ts = dev(s.src), dev(s.dst), dev(s.ts.view(np.int32))
sc = torch.zeros(s.n_edges, dtype=torch.float32, device="cuda")
for _ in range(2):
    ctx.cache_reset()
    ctx.score_stream(src, dst, ts, mc.batch, sc)
torch.cuda.synchronize()
ctx.cache_reset()
ctx.profile(True)
ctx.score_stream(src, dst, ts, mc.batch, sc)
torch.cuda.synchronize()
st = ctx.profile_read()
ctx.profile(False)
c = ctx.counters()
tg = sum(c[f"l{l}_misses"] for l in range(1, mc.n_layers + 1))
ms, n = st["attn"]
tot = sum(v[0] for v in st.values())
print(f"W={W} attn {ms:.3f} ms over {n} launches ({1e3 * ms / max(1, n):.1f} us avg), targets {tg}, "
      f"{1e6 * ms / max(1, tg):.2f} ns/target; all stages {tot:.2f} ms")
