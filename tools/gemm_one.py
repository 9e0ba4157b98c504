"""Launch one large projection GEMM a few times (for ncu captures).

    python tools/gemm_one.py [prec M N K]
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import make_stream, make_params  # noqa: E402
from paper_conf_ppopp_wangm23_b200 import Context  # noqa: E402

prec, M, N, K = (int(x) for x in (sys.argv[1:5] if len(sys.argv) >= 5 else (3, 5120, 256, 4096)))
s = make_stream("tiny")
ctx = Context.from_stream(s).load_model(make_params(2, 2, s.d_n, s.d_e), n_neighbors=3, max_batch_targets=16,
                                        cache_limit=100, time_window=10)
A = torch.randn(M, K, device="cuda")
B = torch.randn(N, K, device="cuda") / K ** 0.5
C = torch.zeros(M, N, device="cuda")
for _ in range(3):
    ctx.gemm(A, B, C, precision=prec)
torch.cuda.synchronize()
print("ok")
