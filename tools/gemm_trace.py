"""Per-CTA timeline of one tcgen05 GEMM launch inside the pipeline (debug build).

    TG_TRACE=1 python -m paper_conf_ppopp_wangm23_b200.build
    python tools/gemm_trace.py --n 172 --k 1032 [--edges 60000]

Arms the clock64 trace of libtg_trace.so for launches of shape (N, K) (the last
such launch of the run is kept) and prints, in microseconds from each CTA's
entry, the median over CTAs of: setup done, first TMA issue, each k-block's
operands landing at the MMA warp, the final commit, epilogue start/end and exit.
"""
import argparse
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ["TG_LIB"] = os.path.join(ROOT, "paper_conf_ppopp_wangm23_b200", "libtg_trace.so")
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
from synth import make_stream, make_params, get_config  # noqa: E402
from paper_conf_ppopp_wangm23_b200 import Context, TG_PREC_BF16, TG_PREC_TF32, TG_PREC_TF32X3, TG_PREC_F16X3  # noqa: E402
from paper_conf_ppopp_wangm23_b200.tg import lib  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, required=True)
ap.add_argument("--k", type=int, required=True)
ap.add_argument("--edges", type=int, default=60000)
ap.add_argument("--precision", default="bf16")
ap.add_argument("--mode", type=int, default=0)
ap.add_argument("--ghz", type=float, default=1.92)
a = ap.parse_args()
cfg = get_config("reddit")
mc = cfg.model
s = make_stream("reddit", n_edges=a.edges)
flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
prec = {"bf16": TG_PREC_BF16, "tf32": TG_PREC_TF32, "tf32x3": TG_PREC_TF32X3, "f16x3": TG_PREC_F16X3}[a.precision]
ctx = Context.from_stream(s).load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                                        max_batch_targets=2 * mc.batch, cache_limit=mc.cache_limit,
                                        time_window=mc.time_window, precision=prec)
L = lib()
L.tg_debug_tc_trace.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
L.tg_debug_tc_trace(a.n, a.k, a.mode, None)
dev = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
sc = torch.zeros(s.n_edges, dtype=torch.float32, device="cuda")
ctx.score_stream(dev(s.src), dev(s.dst), dev(s.ts.view(np.int32)), mc.batch, sc)
torch.cuda.synchronize()
T = np.zeros((148, 64), dtype=np.int64)
L.tg_debug_tc_trace(0, 0, 0, T.ctypes.data)
live = T[:, 0] != 0
T = T[live]
print(f"CTAs traced: {live.sum()}")
us = lambda c: c / (a.ghz * 1e3)
rel = (T - T[:, :1]).astype(np.float64)
names = {2: "setup", 4: "tma_first", 3: "mma_commit", 5: "epi_start", 6: "epi_end", 7: "exit(t0)",
         55: "exit(w6)", 60: "tma_done", 61: "mma_done", 62 - 0: None}
names = {k: v for k, v in names.items() if v}
names[62] = "epi_done"
for i, nm in names.items():
    v = rel[:, i][T[:, i] != 0]
    if v.size:
        print(f"{nm:11s} median {us(np.median(v)):7.2f} us  min {us(v.min()):7.2f}  max {us(v.max()):7.2f}")
print(f"M {T[0, 63]}")
if a.mode == 3:  # one run: MMA landing (8+kb), producer empty release (24+kb), producer arrive (40+kb)
    for nm, base in (("mma_full", 8), ("prod_empty", 24), ("prod_arrive", 40)):
        med = [us(np.median(rel[:, base + i])) for i in range(16) if (T[:, base + i] != 0).all()]
        print(f"{nm:12s}", " ".join(f"{x:.2f}" for x in med))
if a.mode == 5:  # producer phases per unit: [start, staged, read+issue, converted, empty ok, stored]
    for u in range(8):
        v = [us(np.median(rel[:, 8 + 6 * u + i])) for i in range(6)]
        print(f"unit {u}: " + " ".join(f"{x:7.2f}" for x in v) + "   d: " + " ".join(f"{v[i+1]-v[i]:5.2f}" for i in range(5)))
kb = [i for i in range(8, 55) if (T[:, i] != 0).any()] if a.mode not in (3, 5) else []
if kb:
    med = [us(np.median(rel[:, i])) for i in kb]
    print("k-block landed (median us):", " ".join(f"{x:.2f}" for x in med))
gt = T[:, 1]
print(f"CTA start spread (globaltimer): {(gt.max() - gt.min()) / 1e3:.2f} us")
