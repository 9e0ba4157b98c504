"""GEMM time vs K at one full wave (M = 5120 -> 40 M-tiles x N tiles): per-k-block latency probe."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import make_stream, make_params  # noqa: E402
from paper_conf_ppopp_wangm23_b200 import Context  # noqa: E402

s = make_stream("tiny")
ctx = Context.from_stream(s).load_model(make_params(2, 2, s.d_n, s.d_e), n_neighbors=3, max_batch_targets=16,
                                        cache_limit=100, time_window=10)
M, N = 5120, 256
for prec in (2, 3):
    for K in (64, 256, 512, 1024, 2048, 4096):
        A = torch.randn(M, K, device="cuda")
        B = torch.randn(N, K, device="cuda") / K ** 0.5
        C = torch.zeros(M, N, device="cuda")
        ctx.gemm(A, B, C, precision=prec)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10):
            ctx.gemm(A, B, C, precision=prec)
        e1.record()
        torch.cuda.synchronize()
        us = 1e3 * e0.elapsed_time(e1) / 10
        print(f"prec {prec} K {K:5d}  {us:8.1f} us  {2 * M * N * K / us / 1e6:7.1f} TFLOP/s", flush=True)
