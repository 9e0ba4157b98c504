"""Micro-benchmark of the projection GEMM kernels at the superbatch shapes.

    python tools/gemm_bench.py [--m 6400] [--reps 20]

Times tg_gemm (the library's kernels) with CUDA events; prints TFLOP/s per
(precision, shape). Note tg_gemm re-tiles the weights per call, so timing
uses repeated stream-ordered launches after a warm-up call.
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import make_stream, make_params, get_config  # noqa: E402
from paper_conf_ppopp_wangm23_b200 import Context  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=6400)
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--precs", default="0,1,3,2,4")
a = ap.parse_args()
cfg = get_config("tiny")
s = make_stream("tiny")
ctx = Context.from_stream(s).load_model(make_params(2, 2, s.d_n, s.d_e), n_neighbors=3, max_batch_targets=16,
                                        cache_limit=100, time_window=10)
shapes = [(1032, 172), (516, 1032), (172, 688), (172, 172)]
for prec, name in [(p, {0: "fp32", 1: "tf32x3", 2: "bf16", 3: "tf32", 4: "f16x3"}[p]) for p in map(int, a.precs.split(","))]:
    for N, K in shapes:
        A = torch.randn(a.m, K, device="cuda")
        B = torch.randn(N, K, device="cuda") / K ** 0.5
        C = torch.zeros(a.m, N, device="cuda")
        ctx.gemm(A, B, C, precision=prec)  # warm-up (includes weight tiling on the host)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.reps):   # back-to-back launches, no host sync in between
            ctx.gemm(A, B, C, precision=prec)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.reps
        fl = 2.0 * a.m * N * K
        print(f"{name:7s} M={a.m} N={N:5d} K={K:5d}  {ms * 1e3:9.1f} us  {fl / ms / 1e9:8.1f} TFLOP/s", flush=True)
