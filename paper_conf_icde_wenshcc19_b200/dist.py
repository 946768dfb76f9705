"""Multi-GPU driver: one process per GPU (torchrun), pairs sharded for training, test rows
sharded for prediction, NCCL used only to gather models and probabilities.

Training shards naturally: the k(k-1)/2 binary SVMs are independent, so each
rank trains an LPT-balanced subset of pairs (cost ~ n_p^1.5) with X replicated, and there is
no collective inside the solver loop.  The ranks then combine the disjoint per-pair solutions
(alpha, b, A, B: O(sum n_p) doubles, one all-reduce over NCCL) and every rank rebuilds the
complete model from its own replicated X (gmpsvm_model_from_alpha); serializing and merging
whole partial models (gather_models) remains available.  Prediction shards the test rows
(instances are independent, L273) and all-gathers the m x k probabilities.

NEXT-1 (intra-pair sharding): a pair too costly for one rank -- on MNIST-shaped data one pair
runs 232 outer iterations and bounds pair sharding at ~1.5x on 8 GPUs -- is
trained by every rank at once, its instances split into slices (train_pair_sharded over the
gmpsvm_shard_* calls: per outer iteration one all_gather of the ranks' candidate blocks and one
all-reduce of the working set's f values, O(world * B) doubles).
"""
from __future__ import annotations

import numpy as np

from . import _lib as gm


def pair_list(k):
    return [(s, t) for s in range(k) for t in range(s + 1, k)]


def plan_pairs(class_counts, world, exponent=1.5, only=None):
    """LPT (longest processing time first) assignment of pair indices (all, or `only`) to `world`
    ranks."""
    k = len(class_counts)
    sizes = np.array([class_counts[s] + class_counts[t] for s, t in pair_list(k)], dtype=np.float64)
    order = np.argsort(-(sizes ** exponent), kind="stable")
    if only is not None:
        keep = set(int(p) for p in only)
        order = [p for p in order if int(p) in keep]
    load = np.zeros(world)
    shards = [[] for _ in range(world)]
    for p in order:
        r = int(np.argmin(load))
        shards[r].append(int(p))
        load[r] += sizes[p] ** exponent
    return [sorted(s) for s in shards]


def _backend_device(group=None):
    import torch
    import torch.distributed as dist

    if dist.get_backend(group) == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def all_gather_bytes(buf: np.ndarray, group=None):
    """All-gather variable-length uint8 buffers: sizes first, then padded payloads."""
    import torch
    import torch.distributed as dist

    dev = _backend_device(group)
    world = dist.get_world_size(group)
    n = torch.tensor([buf.size], dtype=torch.int64, device=dev)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    cap = max(sizes)
    payload = torch.zeros(cap, dtype=torch.uint8, device=dev)
    payload[: buf.size] = torch.from_numpy(np.ascontiguousarray(buf)).to(dev)
    outs = [torch.empty(cap, dtype=torch.uint8, device=dev) for _ in range(world)]
    dist.all_gather(outs, payload, group=group)
    return [o[:s].cpu().numpy() for o, s in zip(outs, sizes)]


def gather_models(part: "gm.Model", group=None) -> "gm.Model":
    """Serialize this rank's partial model, all-gather the blobs, merge (identical on all ranks)."""
    blobs = all_gather_bytes(part.serialize(), group)
    parts = [gm.Model.deserialize(b) for b in blobs]
    return gm.Model.merge(parts)


def pair_layout(counts):
    """(pair list, offsets of each pair's alpha in the concatenated pair-local layout)."""
    k = len(counts)
    pairs = pair_list(k)
    sizes = [int(counts[s] + counts[t]) for s, t in pairs]
    return pairs, np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)


def pack_solutions(part: "gm.Model", counts, extra=None):
    """This rank's trained pairs as one flat FP64 vector [alpha | b | A | B | status | trained]
    in the global layout (zeros for pairs other ranks train) -- disjoint across ranks.
    extra: {pair index: train_pair_sharded result} solved outside `part` (rank 0 passes them)."""
    pairs, off = pair_layout(counts)
    P = len(pairs)
    tot = int(off[-1])
    v = np.zeros(tot + 5 * P)
    for p, r in (extra or {}).items():
        v[off[p]:off[p + 1]] = r["alpha"]
        v[tot + p], v[tot + P + p], v[tot + 2 * P + p] = r["b"], r["A"], r["B"]
        v[tot + 3 * P + p] = float(r["status"])
        v[tot + 4 * P + p] = 1.0
    if part is None:  # a rank with no pair (more ranks than pairs): contributes zeros
        return v
    mine = part.trained_pairs()
    for p in mine:
        s, t = pairs[p]
        info = part.pair(s, t, int(counts[s]), int(counts[t]))
        v[off[p]:off[p + 1]] = info["alpha"]
        v[tot + p], v[tot + P + p], v[tot + 2 * P + p] = info["b"], info["A"], info["B"]
        v[tot + 3 * P + p] = float(info["status"])
        v[tot + 4 * P + p] = 1.0
    return v


def gather_solutions(part: "gm.Model", X, y, k, C, gamma, group=None, extra=None, **opts) -> "gm.Model":
    """All-reduce (sum) of the disjoint per-pair solutions, then the complete model rebuilt from
    the local X on every rank (identical on all ranks).  extra: pairs solved by
    train_pair_sharded (identical on every rank: rank 0 contributes them)."""
    import torch
    import torch.distributed as dist

    yy = y.cpu().numpy() if isinstance(y, torch.Tensor) else np.asarray(y)
    counts = np.bincount(yy, minlength=k)
    ex = extra if dist.get_rank(group) == 0 else None
    v = torch.from_numpy(pack_solutions(part, counts, ex)).to(_backend_device(group))
    dist.all_reduce(v, op=dist.ReduceOp.SUM, group=group)
    v = v.cpu().numpy()
    pairs, off = pair_layout(counts)
    P, tot = len(pairs), int(off[-1])
    if not np.all(v[tot + 4 * P:] == 1.0):
        raise RuntimeError("every pair must be trained by exactly one rank")
    return gm.model_from_alpha(X, y, k, C, gamma, v[:tot], v[tot:tot + P], v[tot + P:tot + 2 * P],
                               v[tot + 2 * P:tot + 3 * P], v[tot + 3 * P:tot + 4 * P].astype(np.int32), **opts)


def row_range(m, world, rank):
    lo = (m * rank) // world
    hi = (m * (rank + 1)) // world
    return lo, hi


def all_gather_rows(local, m_total, group=None):
    """All-gather row shards (row_range partition) of a [rows, c] tensor/array into [m_total, c]."""
    import torch
    import torch.distributed as dist

    dev = _backend_device(group)
    world = dist.get_world_size(group)
    t = local if isinstance(local, torch.Tensor) else torch.from_numpy(np.ascontiguousarray(local))
    t = t.to(dev)
    cols = t.shape[1]
    cap = max(row_range(m_total, world, r)[1] - row_range(m_total, world, r)[0] for r in range(world))
    pad = torch.zeros((cap, cols), dtype=t.dtype, device=dev)
    pad[: t.shape[0]] = t
    outs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(outs, pad, group=group)
    pieces = []
    for r in range(world):
        lo, hi = row_range(m_total, world, r)
        pieces.append(outs[r][: hi - lo])
    return torch.cat(pieces, 0)


def _all_gather_f64(x: np.ndarray, group=None):
    """All-gather variable-length FP64 vectors (rank order)."""
    parts = all_gather_bytes(np.frombuffer(np.ascontiguousarray(x, dtype=np.float64).tobytes(), dtype=np.uint8), group)
    return [np.frombuffer(p.tobytes(), dtype=np.float64) for p in parts]


def train_pair_sharded(X, y, k, s, t, C, gamma, eps, group=None, **opts):
    """NEXT-1: pair (s, t) trained by every rank of `group`, its instances sharded (PAPER.md
    L250, L299).  Per outer iteration: candidates -> all_gather -> the same exact selection on
    every rank -> f of the working set all-reduced -> the same local SMO everywhere, f updated
    on each rank's slice.  Returns the pair's alpha (pair-local order), b, A, B, status and
    iteration counts, identical on every rank (and bitwise those of world = 1)."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    dev = _backend_device(group)
    sh = gm.Shard(X, y, k, s, t, C, gamma, eps, rank, world, **opts)
    cand = sh.candidates()
    while True:  # one device round trip per collective
        c = torch.from_numpy(cand).to(dev)
        outs = [torch.empty_like(c) for _ in range(world)]
        dist.all_gather(outs, c, group=group)
        stop, fws = sh.select(torch.stack(outs).cpu().numpy(), want_fws=True)
        if stop:
            break
        fw = torch.from_numpy(fws).to(dev)
        dist.all_reduce(fw, op=dist.ReduceOp.SUM, group=group)
        cand = sh.step(fw.cpu().numpy(), want_cands=True)
    f_full = np.concatenate(_all_gather_f64(sh.f_slice(), group))
    return sh.finish(f_full)


def plan_intra(counts, world, exponent=1.5):
    """Pairs to shard across every rank (NEXT-1): those whose estimated cost (n_p^exponent)
    alone exceeds a rank's even share of the total."""
    k = len(counts)
    sizes = np.array([counts[s] + counts[t] for s, t in pair_list(k)], dtype=np.float64)
    cost = sizes ** exponent
    return [int(p) for p in np.flatnonzero(cost > cost.sum() / world)] if world > 1 else []


def train_predict(X, y, Xt, k, C, gamma, eps, group=None, intra_pairs=None, **opts):
    """Sharded train (pairs) + sharded predict (rows) on every rank; returns (model, prob).
    intra_pairs: pair indices trained by all ranks at once (NEXT-1, train_pair_sharded);
    "auto" = plan_intra; None = none (every pair on one rank)."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    yy = y.cpu().numpy() if isinstance(y, torch.Tensor) else np.asarray(y)
    counts = np.bincount(yy, minlength=k)
    if isinstance(intra_pairs, str):
        intra_pairs = plan_intra(counts, world)
    intra = sorted(int(p) for p in (intra_pairs or []))
    extra = {}
    if intra:
        sopts = {key: opts[key] for key in ("device", "stream", "ws_size", "q", "max_outer_iter") if key in opts}
        pairs = pair_list(k)
        for p in intra:
            extra[p] = train_pair_sharded(X, y, k, pairs[p][0], pairs[p][1], C, gamma, eps, group, **sopts)
    rest = [p for p in range(len(pair_list(k))) if p not in extra]
    mine = plan_pairs(counts, world, only=rest)[rank] if rest else []
    # more ranks than pairs: a rank with an empty shard trains nothing and adds zeros to the
    # all-reduce (the library rejects an empty pair_ids list rather than training every pair)
    part = gm.train(X, y, k, C, gamma, eps, pair_ids=mine, **opts) if mine else None
    dev_opts = {key: opts[key] for key in ("device", "stream", "kernel", "coef0", "degree") if key in opts}
    model = gather_solutions(part, X, y, k, C, gamma, group, extra=extra, **dev_opts)
    model.part_stats = part.train_stats() if part is not None else None  # this rank's training
    m = Xt.shape[0]
    lo, hi = row_range(m, world, rank)
    prob_local = model.predict_proba(Xt[lo:hi])
    prob = all_gather_rows(prob_local, m, group)
    return model, prob
