"""Benchmark: TGAT inference edges/s over a Reddit-shaped stream (BASELINE.json).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config reddit]
                    [--precision fp32|tf32x3|bf16] [--impl ours|reference]

A *step* is one full chronological pass (batches of 200 edges) over
the rank's stream, cold cache (tg_cache_reset, as in the paper's runs), i.e.
the whole hot path S1-S16 per batch. For N > 1 (torchrun, NCCL), one process
per GPU:
  --scaling weak   (default) every rank processes its own Reddit-shaped stream
                   (independent seed): fixed work per GPU;
  --scaling strong the single stream is sharded into contiguous batch ranges
                   [r*nb/N, (r+1)*nb/N) (north_star's deployment).
NCCL only gathers the scores and all-reduces the counters at the end of a
pass; there is no per-batch collective (batches are independent).

--impl reference times the oracle (oracle/, plain float64 CPU TGAT, the
paper's baseline role) on the host cores on a bounded sample of the same
workload (rank 0 only).
"""
import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        d["source"] = "measured (MEASURED_PEAKS.json)"
        return d
    d = dict(PEAKS_FALLBACK)
    d["source"] = "fallback (B200_PROFILING.md)"
    return d


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        self.lines = []
        if self.proc is not None:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                out = ""
            self.lines = [l for l in out.splitlines() if l.strip()]

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in getattr(self, "lines", []):
            f = [x.strip() for x in l.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for n, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


# --------------------------------------------------------- reference arm
def run_reference(args, cfg):
    """The oracle (plain float64 CPU TGAT, no TGOpt optimisations) on host cores."""
    from synth import make_stream, make_params
    from oracle.tgat import Model, TemporalGraph, TGAT
    from threadpoolctl import threadpool_info
    mc = cfg.model
    s = make_stream(args.config)
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    o = TGAT(Model(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e), TemporalGraph(s.n_nodes, s.src, s.dst, s.ts),
             s.node_feat, s.edge_feat, mc.n_neighbors)
    nb = (s.n_edges + mc.batch - 1) // mc.batch
    total = args.warmup + args.steps
    picks = np.linspace(0, nb - 1, total).astype(int)
    times, edges = [], 0
    for i, b in enumerate(picks):
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        t0 = time.perf_counter()
        o.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
            edges += hi - lo
    cores = max([d.get("num_threads", 1) for d in threadpool_info()] + [1])
    val = edges / sum(times)
    sample = f"{args.steps} stratified batches of {mc.batch} edges of the {args.config} stream (1 batch per step)"
    line = {"impl": "reference", "metric": "edges_per_sec", "value": val, "unit": "edges/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * float(np.mean(times)),
            "higher_is_better": True, "scaling": "none", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": args.config, "batch": mc.batch,
                                            "n_layers": mc.n_layers, "k": mc.n_neighbors, "sample": sample},
            "cpu_baseline": {"value": val, "unit": "edges/s", "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def cpu_baseline(cfg, name, seconds=15.0):
    """Oracle edges/s on a bounded sample (rank 0, N = 1): stratified batches until ~`seconds`."""
    from synth import make_stream, make_params
    from oracle.tgat import Model, TemporalGraph, TGAT
    from threadpoolctl import threadpool_info
    mc = cfg.model
    s = make_stream(name)
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    o = TGAT(Model(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e), TemporalGraph(s.n_nodes, s.src, s.dst, s.ts),
             s.node_feat, s.edge_feat, mc.n_neighbors)
    nb = (s.n_edges + mc.batch - 1) // mc.batch
    order = np.linspace(0, nb - 1, 16).astype(int)
    t_all, e_all, used = 0.0, 0, []
    for b in order:
        lo, hi = b * mc.batch, min((b + 1) * mc.batch, s.n_edges)
        t0 = time.perf_counter()
        o.infer_batch(s.src[lo:hi], s.dst[lo:hi], s.ts[lo:hi])
        t_all += time.perf_counter() - t0
        e_all += hi - lo
        used.append(int(b))
        if t_all > seconds:
            break
    cores = max([d.get("num_threads", 1) for d in threadpool_info()] + [1])
    return {"value": e_all / t_all, "unit": "edges/s", "cores": int(cores), "kind": "oracle",
            "sample": f"{len(used)} stratified batches {used} of {mc.batch} edges ({e_all} edges, {t_all:.1f} s)"}


# ---------------------------------------------------------------- main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="reddit")
    ap.add_argument("--precision", default="bf16", choices=["fp32", "tf32x3", "bf16", "tf32"])
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"])
    ap.add_argument("--superbatch", type=int, default=0)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-profile", action="store_true")
    args = ap.parse_args()

    from synth import get_config
    cfg = get_config(args.config)
    mc = cfg.model
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        if rank == 0:
            run_reference(args, cfg)
        return

    import dataclasses
    import torch
    import torch.distributed as dist
    from synth import make_stream, make_params
    from paper_conf_ppopp_wangm23_b200 import (Context, TG_NCOUNTERS, counters_dict, TG_PREC_FP32,
                                              TG_PREC_TF32X3, TG_PREC_BF16, TG_PREC_TF32)
    from paper_conf_ppopp_wangm23_b200.shard import shard_batches, gather_scores, reduce_counters

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    prec = {"fp32": TG_PREC_FP32, "tf32x3": TG_PREC_TF32X3, "bf16": TG_PREC_BF16, "tf32": TG_PREC_TF32}[args.precision]

    if args.scaling == "weak" and world > 1:
        s = make_stream(dataclasses.replace(cfg.stream, seed=cfg.stream.seed + 7919 * rank))
    else:
        s = make_stream(args.config)
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    B = mc.batch
    if args.scaling == "strong":
        b0, b1, e0, e1 = shard_batches(s.n_edges, B, rank, world)
    else:
        b0, b1, e0, e1 = 0, (s.n_edges + B - 1) // B, 0, s.n_edges
    E_rank = e1 - e0
    E_job = s.n_edges if args.scaling == "strong" else s.n_edges * world
    ctx = Context.from_stream(s, device=local)
    ctx.load_model(flat, n_layers=mc.n_layers, n_heads=mc.n_heads, n_neighbors=mc.n_neighbors,
                   max_batch_targets=2 * B, cache_limit=mc.cache_limit, time_window=mc.time_window,
                   precision=prec, superbatch=args.superbatch)
    dev = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    src, dst, ts = dev(s.src[e0:e1]), dev(s.dst[e0:e1]), dev(s.ts[e0:e1].view(np.int32))
    scores = torch.zeros(E_rank, dtype=torch.float32, device="cuda")
    nbr = b1 - b0
    log = torch.zeros(nbr * TG_NCOUNTERS, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")  # > L2 (126 MB)
    stream = torch.cuda.current_stream()

    def collect(sc):
        """End-of-pass NCCL: gather scores, all-reduce the counter vector (north_star)."""
        if world > 1:
            if args.scaling == "strong":
                gather_scores(sc, s.n_edges, B, world, dist, device="cuda")
            else:
                parts = [torch.empty_like(sc) for _ in range(world)]
                dist.all_gather(parts, sc)
            reduce_counters(ctx.counters_raw(), dist, device="cuda")

    def step(sc=scores, a=src, b=dst, c=ts, lg=log):
        ctx.cache_reset()                       # cold cache per pass (paper's protocol)
        ctx.score_stream(a, b, c, B, sc, lg, stream=stream)
        launches = ctx.kernel_launches()
        collect(sc)
        return launches

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    # ---- timed region: K passes, L2 flushed before each, events on the launching stream
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    launches = 0
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for i in range(args.steps):
            flush.zero_()
            ev[i][0].record(stream)
            launches += step()
            ev[i][1].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = [a.elapsed_time(b) for a, b in ev]
    t_rank = sum(ms) / 1e3
    t_max = t_rank
    if world > 1:
        tt = torch.tensor([t_rank], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_max = float(tt.item())
    value = args.steps * E_job / t_max

    # ---- per-batch counters of the last pass (hit rates, dedup ratios)
    lg = log.cpu().numpy().reshape(nbr, TG_NCOUNTERS)
    per = [counters_dict(r, mc.n_layers) for r in lg]
    raw = ctx.counters_raw()  # cumulative since last reset = last pass
    if world > 1:
        raw = reduce_counters(raw, dist, device="cuda")
    tot = counters_dict(raw, mc.n_layers)

    def rate(a, b):
        return a / b if b else None

    hit_mean = float(np.mean([p["l1_hits"] / p["l1_lookups"] for p in per if p["l1_lookups"]]))
    stats = {
        "l1_hit_rate_mean_of_batches": hit_mean,
        "l1_hit_rate_global": rate(tot["l1_hits"], tot["l1_lookups"]),
        "dedup_ratio": {f"l{l}": rate(tot[f"l{l}_n"] - tot[f"l{l}_unique"], tot[f"l{l}_n"])
                        for l in range(1, mc.n_layers + 1)},
        "l0_dup_ratio_na": "layer 0 is not deduplicated (P:L239)",
        "time_table_hit_rate": rate(tot["t_table"], tot["t_table"] + tot["t_direct"]),
        "computed_embeddings": {f"l{l}": tot[f"l{l}_misses"] for l in range(1, mc.n_layers + 1)},
        "cache_evictions": tot["l1_evicted"],
    }

    # ---- e2e: same metric through the public API with pinned HOST buffers
    hs_src = torch.from_numpy(np.ascontiguousarray(s.src[e0:e1])).pin_memory()
    hs_dst = torch.from_numpy(np.ascontiguousarray(s.dst[e0:e1])).pin_memory()
    hs_ts = torch.from_numpy(np.ascontiguousarray(s.ts[e0:e1].view(np.int32))).pin_memory()
    hs_sc = torch.zeros(E_rank, dtype=torch.float32).pin_memory()
    e2e_t = []
    for i in range(args.steps + 1):
        if world > 1:
            dist.barrier()
        flush.zero_()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ctx.cache_reset()
        ctx.score_stream(hs_src, hs_dst, hs_ts, B, hs_sc, None, stream=stream)  # H2D in, D2H out, synced
        collect(hs_sc.cuda(non_blocking=False)) if world > 1 else None
        t1 = time.perf_counter() - t0
        if i:
            e2e_t.append(t1)
    e2e_rank = sum(e2e_t)
    if world > 1:
        tt = torch.tensor([e2e_rank], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e_rank = float(tt.item())
    e2e_val = args.steps * E_job / e2e_rank
    assert np.array_equal(hs_sc.numpy(), scores.cpu().numpy()), "host-buffer path disagrees with device path"

    # ---- per-stage device timing (separate profiled pass of the same workload)
    peaks = load_peaks()
    roof = None
    stages = None
    if not args.no_profile:
        ctx.profile(True)
        ctx.cache_reset()
        ctx.score_stream(src, dst, ts, B, scores, None, stream=stream)
        torch.cuda.synchronize()
        stages = ctx.profile_read()
        ctx.profile(False)
        c = ctx.counters()
        D = s.d_n + s.d_e + s.d_n
        k = mc.n_neighbors
        n_targets = sum(c[f"l{l}_misses"] for l in range(1, mc.n_layers + 1))
        # algorithmic bytes of the attention kernel per computed target:
        # neighbour rows h_j + e_ij, Phi rows (table or computed), u in and c out (2 x H x D),
        # per-slot metadata (row ptr 8 + eid 4 + node 4 + t 4 B)
        per_target = k * (s.d_n + s.d_e) * 4 + k * s.d_n * 4 + 2 * mc.n_heads * D * 4 + k * 20
        attn_ms, attn_n = stages["attn"]
        achieved = (n_targets * per_target) / (attn_ms / 1e3) / 1e9
        traffic = None
        tp = os.path.join(ROOT, "profiles", "attn_traffic_bytes_per_launch.json")
        if os.path.exists(tp):
            traffic = json.load(open(tp)).get(args.config)
        roof = {"kernel": "k_attn", "bound": "hbm", "achieved": achieved, "peak": peaks["hbm_gbs"],
                "unit": "GB/s", "frac": achieved / peaks["hbm_gbs"], "traffic": traffic,
                "peak_source": peaks["source"], "bytes_per_target": per_target, "targets": n_targets,
                "launches": attn_n, "avg_launch_us": 1e3 * attn_ms / max(1, attn_n),
                "stage_share_of_step": attn_ms / max(1e-9, sum(v[0] for v in stages.values()))}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cfg, args.config)

    if rank == 0:
        line = {"metric": "edges_per_sec", "value": value, "unit": "edges/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t_max / args.steps,
                "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
                "dtype": {"fp32": "f32", "tf32x3": "tf32x3", "bf16": "bf16", "tf32": "tf32"}[args.precision],
                "data": "synthetic",
                "config": {"workload": args.config, "n_edges": s.n_edges, "n_nodes": s.n_nodes,
                           "edges_per_rank": E_rank, "batch": B, "n_layers": mc.n_layers, "heads": mc.n_heads,
                           "k": mc.n_neighbors, "d_n": s.d_n, "d_e": s.d_e, "cache_limit": mc.cache_limit,
                           "time_window": mc.time_window, "opts": "dedup+cache+ttable",
                           "superbatch": ctx.superbatch(),
                           "parallelism": (f"independent streams x{world}" if args.scaling == "weak"
                                           else f"batch-range shards x{world}"),
                           "l2": "flushed (256 MB write) before every timed step; inputs > L2",
                           "step": "one cold-cache chronological pass over the rank's batches"},
                "e2e": {"value": e2e_val, "unit": "edges/s", "h2d_bytes_per_step": 12 * E_rank,
                        "d2h_bytes_per_step": 4 * E_rank},
                "gpu_launches": int(launches),
                "roofline": roof, "cpu_baseline": cpu, "clocks": clk.summary(), "stats": stats,
                "stages_ms": {k2: round(v[0], 3) for k2, v in stages.items()} if stages else None,
                "peaks": {k2: peaks[k2] for k2 in ("hbm_gbs", "bf16_tflops", "source") if k2 in peaks}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
