"""Latency probe of the projection GEMM: time vs M at small N, K (back-to-back launches)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import make_stream, make_params  # noqa: E402
from paper_conf_ppopp_wangm23_b200 import Context  # noqa: E402

s = make_stream("tiny")
ctx = Context.from_stream(s).load_model(make_params(2, 2, s.d_n, s.d_e), n_neighbors=3, max_batch_targets=16,
                                        cache_limit=100, time_window=10)
for prec in (2, 0):
    for (M, N, K) in [(128, 16, 64), (128, 96, 64), (128, 176, 172), (1024, 176, 172), (6400, 176, 172),
                      (128, 208, 1032), (6400, 208, 1032)]:
        A = torch.randn(M, K, device="cuda")
        B = torch.randn(N, K, device="cuda")
        C = torch.zeros(M, N, device="cuda")
        ctx.gemm(A, B, C, precision=prec)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            ctx.gemm(A, B, C, precision=prec)
        e1.record()
        torch.cuda.synchronize()
        print(prec, M, N, K, "%.1f us" % (1e3 * e0.elapsed_time(e1) / 20), flush=True)
