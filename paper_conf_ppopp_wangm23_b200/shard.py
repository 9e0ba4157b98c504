"""Batch-range sharding over GPUs (north_star: "sharding contiguous batch ranges
of the stream").

Each rank holds a replica of the graph and weights and its own memo cache and
processes the contiguous batch range [floor(r*nb/G), floor((r+1)*nb/G)). There
is no data-path collective: every batch's scores are a pure function of
(graph, weights, batch). At the end of a pass NCCL gathers the scores
(padded to the largest shard) and all-reduces the int64 counter vector.
Host-side logic only; the per-rank work runs through libtg.
"""
import numpy as np


def shard_batches(n_edges: int, batch: int, rank: int, world: int):
    """(first batch, end batch, first edge, end edge) of rank `rank`."""
    nb = (n_edges + batch - 1) // batch
    b0 = (rank * nb) // world
    b1 = ((rank + 1) * nb) // world
    return b0, b1, b0 * batch, min(b1 * batch, n_edges)


def max_shard_edges(n_edges: int, batch: int, world: int):
    return max(e1 - e0 for (_, _, e0, e1) in (shard_batches(n_edges, batch, r, world) for r in range(world)))


def gather_scores(local_scores, n_edges: int, batch: int, world: int, dist, device=None):
    """All-gather every rank's scores into the full [n_edges] vector (rank order = stream order)."""
    import torch
    pad = max_shard_edges(n_edges, batch, world)
    buf = torch.zeros(pad, dtype=torch.float32, device=device)
    buf[: local_scores.numel()] = local_scores
    parts = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(parts, buf)
    out = []
    for r in range(world):
        _, _, e0, e1 = shard_batches(n_edges, batch, r, world)
        out.append(parts[r][: e1 - e0])
    return torch.cat(out)


def reduce_counters(counters: np.ndarray, dist, device=None):
    """SUM all-reduce of the int64 counter vector (tg_counters_read layout)."""
    import torch
    t = torch.as_tensor(np.asarray(counters, np.int64), device=device)
    dist.all_reduce(t)
    return t.cpu().numpy()
