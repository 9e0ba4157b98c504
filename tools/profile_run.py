"""One cold-cache pass over a stream through the C ABI, for ncu captures.

    python tools/profile_run.py [--config reddit] [--precision bf16] [--edges N]
"""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import make_stream, make_params, get_config  # noqa: E402
from paper_conf_ppopp_wangm23_b200 import (Context, TG_PREC_FP32, TG_PREC_TF32X3, TG_PREC_BF16, TG_PREC_TF32,  # noqa: E402
                                          TG_PREC_F16X3)

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="reddit")
ap.add_argument("--precision", default="bf16")
ap.add_argument("--edges", type=int, default=None)
ap.add_argument("--superbatch", type=int, default=0)
a = ap.parse_args()
cfg = get_config(a.config)
mc = cfg.model
s = make_stream(a.config, n_edges=a.edges)
flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
prec = {"fp32": TG_PREC_FP32, "tf32x3": TG_PREC_TF32X3, "bf16": TG_PREC_BF16, "tf32": TG_PREC_TF32,
        "f16x3": TG_PREC_F16X3}[a.precision]
ctx = Context.from_stream(s).load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                                        max_batch_targets=2 * mc.batch, cache_limit=mc.cache_limit,
                                        time_window=mc.time_window, precision=prec, superbatch=a.superbatch)
dev = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
sc = torch.zeros(s.n_edges, dtype=torch.float32, device="cuda")
ctx.score_stream(dev(s.src), dev(s.dst), dev(s.ts.view(np.int32)), mc.batch, sc)
torch.cuda.synchronize()
print("launches", ctx.kernel_launches(), "l1 hits", ctx.counters()["l1_hits"])
