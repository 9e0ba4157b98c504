"""Thin ctypes binding of libtg.so (include/tg.h). Argument marshalling only:
every step of the hot path runs in the library's sm_100a kernels. There is no
CPU fallback: if libtg.so is missing or the device is absent, calls raise.

Arrays may be torch tensors (CUDA -> device pointer, CPU -> host pointer) or
numpy arrays (host pointer); the library detects the memory space.
"""
import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TG_LIB") or os.path.join(_PKG, "libtg.so")

TG_OPT_DEDUP, TG_OPT_CACHE, TG_OPT_TTABLE, TG_OPT_ALL, TG_OPT_HOST_CACHE = 1, 2, 4, 7, 8
TG_PREC_FP32, TG_PREC_TF32X3, TG_PREC_BF16, TG_PREC_TF32, TG_PREC_F16X3 = 0, 1, 2, 3, 4
TG_MAX_LAYERS = 4
TG_CNT_PER_LAYER = 6
TG_CNT_TTABLE = (TG_MAX_LAYERS + 1) * TG_CNT_PER_LAYER
TG_CNT_TDIRECT = TG_CNT_TTABLE + 1
TG_NCOUNTERS = TG_CNT_TDIRECT + 1
COUNTER_FIELDS = ("n", "unique", "lookups", "hits", "misses", "evicted")

EXPORTS = ("tg_graph_load", "tg_model_load", "tg_embed_batch", "tg_score_edges", "tg_score_stream",
           "tg_score_stream_neg",
           "tg_score_pairs", "tg_cache_reset", "tg_counters_read", "tg_dedup", "tg_sample", "tg_time_encode",
           "tg_kernel_launches", "tg_free", "tg_strerror", "tg_version", "tg_profile_enable",
           "tg_profile_read", "tg_gemm", "tg_superbatch")
STAGES = ("prep", "dedup", "lookup", "sample", "resolve", "proj_k", "attn", "proj_v", "lnorm", "ffn1", "ffn2",
          "score", "other", "phi")


class TGError(RuntimeError):
    pass


class GraphDesc(ctypes.Structure):
    _fields_ = [("n_nodes", ctypes.c_int64), ("n_edges", ctypes.c_int64),
                ("src", ctypes.c_void_p), ("dst", ctypes.c_void_p), ("ts", ctypes.c_void_p),
                ("node_feat", ctypes.c_void_p), ("d_n", ctypes.c_int32),
                ("edge_feat", ctypes.c_void_p), ("d_e", ctypes.c_int32)]


class ModelCfg(ctypes.Structure):
    _fields_ = [("n_layers", ctypes.c_int32), ("n_heads", ctypes.c_int32), ("n_neighbors", ctypes.c_int32),
                ("d_t", ctypes.c_int32), ("max_batch_targets", ctypes.c_int32),
                ("cache_limit", ctypes.c_int64), ("time_window", ctypes.c_int32),
                ("opts", ctypes.c_uint32), ("precision", ctypes.c_int32), ("superbatch", ctypes.c_int32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise TGError(f"{LIB_PATH} missing: run __graft_entry__.build() "
                          "(python -m paper_conf_ppopp_wangm23_b200.build); there is no fallback")
        L = ctypes.CDLL(LIB_PATH)
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
        L.tg_graph_load.argtypes = [ctypes.c_int, ctypes.POINTER(GraphDesc), ctypes.POINTER(vp)]
        L.tg_model_load.argtypes = [vp, ctypes.POINTER(ModelCfg), vp, i64]
        L.tg_embed_batch.argtypes = [vp, vp, vp, i64, vp, vp]
        L.tg_score_edges.argtypes = [vp, vp, vp, vp, i64, vp, vp]
        L.tg_score_stream.argtypes = [vp, vp, vp, vp, i64, i32, vp, vp, vp]
        L.tg_score_stream_neg.argtypes = [vp, vp, vp, vp, vp, i64, i32, vp, vp, vp]
        L.tg_score_pairs.argtypes = [vp, vp, vp, i64, vp, vp, i64, vp, vp]
        L.tg_cache_reset.argtypes = [vp, i64]
        L.tg_counters_read.argtypes = [vp, vp, i32]
        L.tg_dedup.argtypes = [vp, vp, vp, i64, vp, vp, vp, vp, vp]
        L.tg_sample.argtypes = [vp, vp, vp, i64, vp, vp, vp, vp]
        L.tg_time_encode.argtypes = [vp, vp, i64, i32, vp, vp]
        L.tg_profile_enable.argtypes = [vp, i32]
        L.tg_profile_read.argtypes = [vp, vp, vp, i32]
        L.tg_gemm.argtypes = [vp, i32, i32, i32, i32, vp, vp, vp, i32, vp, vp]
        L.tg_kernel_launches.argtypes = [vp]
        L.tg_kernel_launches.restype = i64
        L.tg_superbatch.argtypes = [vp]
        L.tg_superbatch.restype = i32
        L.tg_free.argtypes = [vp]
        L.tg_free.restype = None
        L.tg_strerror.argtypes = [ctypes.c_int]
        L.tg_strerror.restype = ctypes.c_char_p
        L.tg_version.restype = ctypes.c_char_p
        for f in ("tg_graph_load", "tg_model_load", "tg_embed_batch", "tg_score_edges", "tg_score_stream",
                  "tg_score_pairs", "tg_cache_reset", "tg_counters_read", "tg_dedup", "tg_sample", "tg_time_encode",
                  "tg_profile_enable", "tg_profile_read", "tg_gemm"):
            getattr(L, f).restype = ctypes.c_int
        _lib = L
    return _lib


def _check(status, what):
    if status != 0:
        msg = lib().tg_strerror(status).decode()
        raise TGError(f"{what}: {msg} ({status})")


def _ptr(a):
    """Raw address of a torch tensor or a C-contiguous numpy array (None -> NULL)."""
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        if not a.is_contiguous():
            raise TGError("tensor must be contiguous")
        return a.data_ptr()
    if isinstance(a, np.ndarray):
        if not a.flags["C_CONTIGUOUS"]:
            raise TGError("array must be C-contiguous")
        return a.ctypes.data
    raise TGError(f"unsupported buffer type {type(a)}")


def _stream(stream):
    if stream is None:
        try:
            import torch
            return torch.cuda.current_stream().cuda_stream
        except Exception:  # no torch / no device: legacy default stream
            return None
    if hasattr(stream, "cuda_stream"):
        return stream.cuda_stream
    return int(stream)


class Context:
    """One device context: graph + model + memo cache (tg_graph_load / tg_model_load)."""

    def __init__(self, n_nodes, src, dst, ts, node_feat, edge_feat, device=0):
        self._keep = [np.ascontiguousarray(src, np.int32), np.ascontiguousarray(dst, np.int32),
                      np.ascontiguousarray(ts, np.uint32), np.ascontiguousarray(node_feat, np.float32),
                      np.ascontiguousarray(edge_feat, np.float32)]
        s, d, t, X, E = self._keep
        desc = GraphDesc(int(n_nodes), int(s.size), _ptr(s), _ptr(d), _ptr(t), _ptr(X), int(X.shape[1]),
                         _ptr(E), int(E.shape[1]))
        h = ctypes.c_void_p()
        _check(lib().tg_graph_load(int(device), ctypes.byref(desc), ctypes.byref(h)), "tg_graph_load")
        self.h = h
        self.d_n = int(X.shape[1])
        self.d_e = int(E.shape[1])
        self._keep = None  # the library copied everything
        self.cfg = None

    @classmethod
    def from_stream(cls, stream, device=0):
        return cls(stream.n_nodes, stream.src, stream.dst, stream.ts, stream.node_feat, stream.edge_feat, device)

    def load_model(self, params, n_layers=2, n_heads=2, n_neighbors=20, d_t=None, max_batch_targets=400,
                   cache_limit=2_000_000, time_window=10_000, opts=TG_OPT_ALL, precision=TG_PREC_FP32,
                   superbatch=0):
        d_t = self.d_n if d_t is None else d_t
        p = np.ascontiguousarray(params, np.float32)
        cfg = ModelCfg(n_layers, n_heads, n_neighbors, d_t, max_batch_targets, cache_limit, time_window,
                       opts, precision, superbatch)
        _check(lib().tg_model_load(self.h, ctypes.byref(cfg), _ptr(p), p.size), "tg_model_load")
        self.cfg = cfg
        return self

    def embed_batch(self, nodes, ts, out, stream=None):
        _check(lib().tg_embed_batch(self.h, _ptr(nodes), _ptr(ts), int(nodes.shape[0]), _ptr(out),
                                    _stream(stream)), "tg_embed_batch")
        return out

    def score_edges(self, src, dst, ts, scores, stream=None):
        _check(lib().tg_score_edges(self.h, _ptr(src), _ptr(dst), _ptr(ts), int(src.shape[0]), _ptr(scores),
                                    _stream(stream)), "tg_score_edges")
        return scores

    def score_pairs(self, nodes, ts, pair_a, pair_b, scores, stream=None):
        _check(lib().tg_score_pairs(self.h, _ptr(nodes), _ptr(ts), int(nodes.shape[0]), _ptr(pair_a), _ptr(pair_b),
                                    int(pair_a.shape[0]), _ptr(scores), _stream(stream)), "tg_score_pairs")
        return scores

    def score_stream(self, src, dst, ts, batch, scores, batch_counters=None, stream=None):
        _check(lib().tg_score_stream(self.h, _ptr(src), _ptr(dst), _ptr(ts), int(src.shape[0]), int(batch),
                                     _ptr(scores), _ptr(batch_counters), _stream(stream)), "tg_score_stream")
        return scores

    def score_stream_neg(self, src, dst, ts, neg, batch, scores, batch_counters=None, stream=None):
        """scores[:E] = positive (src, dst) pairs, scores[E:] = (src, neg) pairs (NEXT-3)."""
        _check(lib().tg_score_stream_neg(self.h, _ptr(src), _ptr(dst), _ptr(ts), _ptr(neg), int(src.shape[0]),
                                         int(batch), _ptr(scores), _ptr(batch_counters), _stream(stream)),
               "tg_score_stream_neg")
        return scores

    def cache_reset(self, new_limit=-1):
        _check(lib().tg_cache_reset(self.h, int(new_limit)), "tg_cache_reset")

    def counters_raw(self):
        out = np.zeros(TG_NCOUNTERS, np.int64)
        _check(lib().tg_counters_read(self.h, out.ctypes.data, TG_NCOUNTERS), "tg_counters_read")
        return out

    def counters(self):
        return counters_dict(self.counters_raw(), self.cfg.n_layers)

    def dedup(self, nodes, ts, uniq_nodes, uniq_ts, inv, n_uniq, stream=None):
        _check(lib().tg_dedup(self.h, _ptr(nodes), _ptr(ts), int(nodes.shape[0]), _ptr(uniq_nodes),
                              _ptr(uniq_ts), _ptr(inv), _ptr(n_uniq), _stream(stream)), "tg_dedup")

    def sample(self, nodes, ts, nbr, eid, nts, stream=None):
        _check(lib().tg_sample(self.h, _ptr(nodes), _ptr(ts), int(nodes.shape[0]), _ptr(nbr), _ptr(eid),
                               _ptr(nts), _stream(stream)), "tg_sample")

    def time_encode(self, delta, out, use_table=True, stream=None):
        _check(lib().tg_time_encode(self.h, _ptr(delta), int(delta.shape[0]), int(bool(use_table)), _ptr(out),
                                    _stream(stream)), "tg_time_encode")

    def profile(self, on=True):
        _check(lib().tg_profile_enable(self.h, int(bool(on))), "tg_profile_enable")

    def profile_read(self):
        ms = np.zeros(len(STAGES), np.float64)
        cnt = np.zeros(len(STAGES), np.int64)
        _check(lib().tg_profile_read(self.h, ms.ctypes.data, cnt.ctypes.data, len(STAGES)), "tg_profile_read")
        return {s: (float(m), int(c)) for s, m, c in zip(STAGES, ms, cnt)}

    def gemm(self, A, B, C, bias=None, relu=False, precision=TG_PREC_FP32, stream=None):
        """C = A B^T (+bias, ReLU) with the library's dense-projection kernels (unit entry)."""
        M, K = A.shape
        N = B.shape[0]
        _check(lib().tg_gemm(self.h, int(precision), int(M), int(N), int(K), _ptr(A), _ptr(B), _ptr(bias),
                             int(bool(relu)), _ptr(C), _stream(stream)), "tg_gemm")
        return C

    def kernel_launches(self):
        return int(lib().tg_kernel_launches(self.h))

    def superbatch(self):
        """S in use by score_stream (after the default and the capacity clamp)."""
        return int(lib().tg_superbatch(self.h))

    def close(self):
        if getattr(self, "h", None):
            lib().tg_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def counters_dict(raw, n_layers):
    out = {}
    for l in range(n_layers + 1):
        for j, f in enumerate(COUNTER_FIELDS):
            out[f"l{l}_{f}"] = int(raw[l * TG_CNT_PER_LAYER + j])
    out["t_table"] = int(raw[TG_CNT_TTABLE])
    out["t_direct"] = int(raw[TG_CNT_TDIRECT])
    return out


def version():
    return lib().tg_version().decode()
