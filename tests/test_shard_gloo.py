"""Multi-process (gloo, world_size 2, CPU) checks of the batch-range sharding and
the end-of-pass gathers used by bench.py for N > 1 GPUs.

The per-rank compute is replaced by the oracle's Alg. 1 simulator on CPU
(counters) and by a deterministic per-batch stand-in for the scores, so only
the host logic is exercised: partition, score all-gather order, counter
all-reduce = sum over shards of the per-shard (cold-cache) simulation.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_wangm23_b200.shard import shard_batches, gather_scores, reduce_counters


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_shards_partition_the_stream():
    for E, B, G in [(10_000, 200, 1), (10_000, 200, 3), (672_447, 200, 8), (5, 200, 4), (1001, 7, 5)]:
        edges = []
        for r in range(G):
            b0, b1, e0, e1 = shard_batches(E, B, r, G)
            assert e0 == b0 * B and e1 <= E
            edges.append((e0, e1))
        assert edges[0][0] == 0 and edges[-1][1] == E
        for (a0, a1), (c0, c1) in zip(edges, edges[1:]):
            assert a1 == c0
        sizes = [e1 - e0 for e0, e1 in edges]
        assert max(sizes) - min(sizes) <= B + (E % B)


def _worker(rank, world, port, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import torch
    from synth import make_stream, make_params, get_config
    from oracle.tgat import Model, TemporalGraph, TGAT
    from oracle.tgopt import TGOptSim
    cfg = get_config("tiny_bip")
    mc = cfg.model
    s = make_stream("tiny_bip")
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    o = TGAT(Model(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e), TemporalGraph(s.n_nodes, s.src, s.dst, s.ts),
             s.node_feat, s.edge_feat, mc.n_neighbors)
    b0, b1, e0, e1 = shard_batches(s.n_edges, mc.batch, rank, world)
    sim = TGOptSim(o, cache_limit=mc.cache_limit, time_window=mc.time_window, compute=False)  # own cold cache
    for lo in range(e0, e1, mc.batch):
        sim.infer_batch(s.src[lo:lo + mc.batch], s.dst[lo:lo + mc.batch], s.ts[lo:lo + mc.batch])
    c = sim.counters()
    keys = sorted(c)
    local = np.array([c[k] for k in keys], np.int64)
    total = reduce_counters(local, dist)
    scores = torch.arange(e0, e1, dtype=torch.float32) * 0.5   # stand-in: a pure function of the edge
    full = gather_scores(scores, s.n_edges, mc.batch, world, dist)
    if rank == 0:
        out_q.put((keys, total.tolist(), full.numpy().tolist()))
    dist.destroy_process_group()


def test_gloo_world2_gathers_match_sequential_shards():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    keys, total, full = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    from synth import make_stream, make_params, get_config
    from oracle.tgat import Model, TemporalGraph, TGAT
    from oracle.tgopt import TGOptSim
    cfg = get_config("tiny_bip")
    mc = cfg.model
    s = make_stream("tiny_bip")
    flat = make_params(mc.n_layers, mc.n_heads, s.d_n, s.d_e)
    o = TGAT(Model(flat, mc.n_layers, mc.n_heads, s.d_n, s.d_e), TemporalGraph(s.n_nodes, s.src, s.dst, s.ts),
             s.node_feat, s.edge_feat, mc.n_neighbors)
    want = np.zeros(len(keys), np.int64)
    for r in range(world):
        _, _, e0, e1 = shard_batches(s.n_edges, mc.batch, r, world)
        sim = TGOptSim(o, cache_limit=mc.cache_limit, time_window=mc.time_window, compute=False)
        for lo in range(e0, e1, mc.batch):
            sim.infer_batch(s.src[lo:lo + mc.batch], s.dst[lo:lo + mc.batch], s.ts[lo:lo + mc.batch])
        c = sim.counters()
        want += np.array([c[k] for k in keys], np.int64)
    assert total == want.tolist()
    assert np.array_equal(np.array(full), np.arange(s.n_edges, dtype=np.float32) * 0.5)
    # per-shard cold caches: the sharded run misses at least as often as one shard
    single = TGOptSim(o, cache_limit=mc.cache_limit, time_window=mc.time_window, compute=False)
    for lo in range(0, s.n_edges, mc.batch):
        single.infer_batch(s.src[lo:lo + mc.batch], s.dst[lo:lo + mc.batch], s.ts[lo:lo + mc.batch])
    assert total[keys.index("l1_misses")] >= single.counters()["l1_misses"]


def test_bench_spawns_one_rank_per_gpu():
    """bench.py --gpus N without a torchrun environment re-executes itself through
    torch.distributed.run with N local ranks (127.0.0.1); under torchrun WORLD_SIZE must
    equal --gpus (--gpus used to be ignored)."""
    import bench
    cmd = bench.spawn_cmd(["--gpus", "4", "--steps", "2"], 4, 29555)
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in cmd and "--master-addr=127.0.0.1" in cmd and "--master-port=29555" in cmd
    assert cmd[-3:] == ["--gpus", "4", "--steps", "2"][-3:] and cmd[cmd.index("--master-port=29555") + 1].endswith("bench.py")
    assert bench.check_world("0", 1) == 1 and bench.check_world("8", 8) == 8
    with pytest.raises(SystemExit):
        bench.check_world("2", 8)
    with pytest.raises(SystemExit):
        bench.check_world("0", 2)
