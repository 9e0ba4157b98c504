"""Run the bench workload's stream pass several times (device buffers, then host buffers) and
report whether the scores are bit-identical (every kernel is meant to be deterministic)."""
import sys, os
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests.gpu_helpers import setup, make_ctx
cfg, s, flat = setup(sys.argv[1] if len(sys.argv) > 1 else "reddit")
mc = cfg.model
prec = int(sys.argv[2]) if len(sys.argv) > 2 else 1
ctx = make_ctx(s, flat, mc, precision=prec)
d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
outs = []
for r in range(3):
    sc = torch.zeros(s.n_edges, dtype=torch.float32, device="cuda")
    ctx.cache_reset()
    ctx.score_stream(d(s.src), d(s.dst), d(s.ts.view(np.int32)), mc.batch, sc)
    torch.cuda.synchronize()
    outs.append(sc.cpu().numpy())
hs = np.zeros(s.n_edges, np.float32)
ctx.cache_reset()
ctx.score_stream(s.src, s.dst, s.ts.view(np.int32), mc.batch, hs)
outs.append(hs)
for i in range(1, len(outs)):
    diff = np.flatnonzero(outs[i] != outs[0])
    print(i, "identical" if diff.size == 0 else f"{diff.size} differ, first at edge {diff[0]} (batch {diff[0] // mc.batch}), max {np.abs(outs[i]-outs[0]).max():.3e}")
