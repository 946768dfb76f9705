"""Multi-process host plumbing of the multi-GPU path on CPU (gloo, world_size 2):
LPT pair sharding, variable-size model-blob all_gather + merge through libgmpsvm's host
code, and the test-row shard all_gather.  The NCCL path differs only in the backend."""
import ctypes as ct
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from blobfmt import make_blob, pair_list


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _problem(k=4):
    rng = np.random.default_rng(0)
    n, d = 60, 5
    X = rng.normal(size=(n, d)).astype(np.float32)
    y = (np.arange(n) % k).astype(np.int32)
    rng.shuffle(y)
    counts = np.bincount(y, minlength=k)
    pairs = pair_list(k)
    P = len(pairs)
    alphas = {}
    for p, (s, t) in enumerate(pairs):
        a = rng.uniform(0, 1, size=counts[s] + counts[t])
        a[rng.random(len(a)) < 0.5] = 0.0
        alphas[p] = a
    b, A, B = rng.normal(size=P), -rng.uniform(1, 2, size=P), rng.normal(size=P)
    return X, y, k, alphas, b, A, B


def _worker(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_icde_wenshcc19_b200 as gm
        from paper_conf_icde_wenshcc19_b200 import dist as gdist

        X, y, k, alphas, b, A, B = _problem()
        shards = gdist.plan_pairs(np.bincount(y, minlength=k), world)
        mine = {p: alphas[p] for p in shards[rank]}
        ssz = ct.sizeof(gm._lib.TrainStats)
        blob, perm, _ = make_blob(X, y, k, 1.0, 0.5, 1e-3, mine, b, A, B, ssz)
        part = gm.Model.deserialize(blob)
        merged = gdist.gather_models(part)
        full_blob, _, sv_pos = make_blob(X, y, k, 1.0, 0.5, 1e-3, alphas, b, A, B, ssz)
        expect = gm.Model.deserialize(full_blob)
        ok = merged.n_pairs_trained == len(pair_list(k)) and merged.n_sv == expect.n_sv
        ok &= bool(np.array_equal(merged.sv_index(), expect.sv_index()))
        counts = np.bincount(y, minlength=k)
        for p, (s, t) in enumerate(pair_list(k)):
            info = merged.pair(s, t, int(counts[s]), int(counts[t]))
            ok &= bool(np.array_equal(info["alpha"], alphas[p])) and info["b"] == b[p] and info["A"] == A[p]
        # byte-identical merged blob on every rank
        blobs = gdist.all_gather_bytes(merged.serialize())
        ok &= all(np.array_equal(blobs[0], x) for x in blobs)
        # test-row shards
        m = 11
        lo, hi = gdist.row_range(m, world, rank)
        local = np.arange(lo * 3, hi * 3, dtype=np.float64).reshape(hi - lo, 3)
        allp = gdist.all_gather_rows(local, m).numpy()
        ok &= bool(np.array_equal(allp, np.arange(m * 3, dtype=np.float64).reshape(m, 3)))
        q.put((rank, bool(ok), ""))
    except Exception as e:  # report instead of hanging the parent
        q.put((rank, False, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _pack_worker(rank, world, port, q):
    """pack_solutions + the all-reduce of dist.gather_solutions with more ranks than pairs
    (k = 3: P = 3 < world = 4): the empty shard contributes zeros; the reduced vector holds every
    pair exactly once, in the global [alpha | b | A | B | status | trained] layout."""
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_icde_wenshcc19_b200 as gm
        from paper_conf_icde_wenshcc19_b200 import dist as gdist

        X, y, k, alphas, b, A, B = _problem(k=3)
        counts = np.bincount(y, minlength=k)
        shards = gdist.plan_pairs(counts, world)
        mine = shards[rank]
        ssz = ct.sizeof(gm._lib.TrainStats)
        part = None
        if mine:
            blob, _, _ = make_blob(X, y, k, 1.0, 0.5, 1e-3, {p: alphas[p] for p in mine}, b, A, B, ssz)
            part = gm.Model.deserialize(blob)
        v = torch.from_numpy(gdist.pack_solutions(part, counts))
        dist.all_reduce(v, op=dist.ReduceOp.SUM)
        v = v.numpy()
        pairs, off = gdist.pair_layout(counts)
        P, tot = len(pairs), int(off[-1])
        ok = sum(1 for s in shards if not s) == world - P
        ok &= bool(np.all(v[tot + 4 * P:] == 1.0))
        for p in range(P):
            ok &= bool(np.array_equal(v[off[p]:off[p + 1]], alphas[p]))
        ok &= bool(np.array_equal(v[tot:tot + P], b) and np.array_equal(v[tot + P:tot + 2 * P], A))
        ok &= bool(np.array_equal(v[tot + 2 * P:tot + 3 * P], B))
        q.put((rank, bool(ok), ""))
    except Exception as e:
        q.put((rank, False, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _run(target, world):
    import __graft_entry__

    __graft_entry__.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=target, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert all(ok for _, ok, _ in res), res


def test_gloo_world4_pack_solutions_more_ranks_than_pairs():
    _run(_pack_worker, 4)


def test_plan_pairs_lpt_covers_all_pairs():
    from paper_conf_icde_wenshcc19_b200 import dist as gdist

    counts = np.array([6000, 6100, 5900, 6050, 5950, 6010, 5990, 6020, 5980, 6000])
    for world in (1, 2, 4, 8):
        shards = gdist.plan_pairs(counts, world)
        flat = sorted(p for s in shards for p in s)
        assert flat == list(range(45))
        loads = [sum((counts[a] + counts[b]) ** 1.5 for a, b in (pair_list(10)[p] for p in s)) for s in shards]
        assert max(loads) / (sum(loads) / world) < 1.2


def test_gloo_world2_gather_merge():
    import __graft_entry__

    __graft_entry__.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert all(ok for _, ok, _ in res), res


# ------------------------------------------------------------------------------------ NEXT-1
def _ord_key(f):
    """Order-preserving uint64 key of FP64 values (negative: all bits flipped; else sign set)."""
    u = np.asarray(f, dtype=np.float64).view(np.uint64)
    neg = (u >> np.uint64(63)) == 1
    return np.where(neg, ~u, u | np.uint64(1 << 63))


def _cand_block(f, a, y, C, ret, lo, hi, need, m):
    """A rank's candidate block (layout of gmpsvm_shard_merge) from its slice [lo, hi), numpy."""
    blk = np.zeros(4 + 4 * m)
    idx = np.arange(lo, hi)
    iu = ((y[idx] > 0) & (a[idx] < C)) | ((y[idx] < 0) & (a[idx] > 0))
    il = ((y[idx] > 0) & (a[idx] > 0)) | ((y[idx] < 0) & (a[idx] < C))
    blk[0] = f[idx][iu].min() if iu.any() else np.finfo(np.float64).max
    blk[1] = f[idx][il].max() if il.any() else -np.finfo(np.float64).max
    cu = idx[iu & ~ret[idx]]
    cl = idx[il & ~ret[idx]]
    cu = cu[np.lexsort((cu, f[cu]))][:need]       # smallest f, lowest index on ties
    cl = cl[np.lexsort((cl, -f[cl]))][:need]      # largest f, lowest index on ties
    blk[2], blk[3] = len(cu), len(cl)
    blk[4:4 + len(cu)] = _ord_key(f[cu]).view(np.float64)
    blk[4 + m:4 + m + len(cu)] = cu
    blk[4 + 2 * m:4 + 2 * m + len(cl)] = (~_ord_key(f[cl])).view(np.float64)
    blk[4 + 3 * m:4 + 3 * m + len(cl)] = cl
    return blk


def _reference_selection(f, a, y, C, ret, need, need_u):
    """Reading R19 on the whole vector: need_u smallest f in I_u \\ retained, then the largest f in
    I_l \\ retained not taken, then I_u again if I_l ran short (ties: lowest index)."""
    n = len(f)
    idx = np.arange(n)
    iu = (((y > 0) & (a < C)) | ((y < 0) & (a > 0))) & ~ret
    il = (((y > 0) & (a > 0)) | ((y < 0) & (a < C))) & ~ret
    U = idx[iu][np.lexsort((idx[iu], f[iu]))]
    L = idx[il][np.lexsort((idx[il], -f[il]))]
    picks = list(U[:need_u])
    for j in L:
        if len(picks) >= need:
            break
        if j not in picks:
            picks.append(j)
    for j in U[need_u:]:
        if len(picks) >= need:
            break
        if j not in picks:
            picks.append(j)
    gap = f[(((y > 0) & (a > 0)) | ((y < 0) & (a < C)))].max() - f[(((y > 0) & (a < C)) | ((y < 0) & (a > 0)))].min()
    return np.array(picks, dtype=np.int32), gap


def _merge_worker(rank, world, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_icde_wenshcc19_b200 as gm

        ok = True
        for seed in range(6):
            rng = np.random.default_rng(seed)
            n, C, B = 1500, 1.0, 96
            y = np.where(np.arange(n) < 700, 1, -1)
            a = np.where(rng.random(n) < 0.4, 0.0, np.where(rng.random(n) < 0.5, C, rng.uniform(0, C, n)))
            f = np.round(rng.normal(0, 1, n), 2 if seed % 2 else 9)  # seed odd: many exact ties
            ret = np.zeros(n, dtype=bool)
            ret[rng.choice(n, size=B // 2, replace=False)] = True
            need = B - int(ret.sum())
            if seed == 5:  # I_l almost empty: the selection takes I_u again
                a[:700] = 0.0
                a[700:] = C
                a[700:705] = 0.5
            per = -(-n // world)
            lo, hi = min(n, rank * per), min(n, rank * per + per)
            blk = torch.from_numpy(_cand_block(f, a, y, C, ret, lo, hi, need, B))
            outs = [torch.empty_like(blk) for _ in range(world)]
            dist.all_gather(outs, blk)
            picks, gap = gm.shard_merge(torch.stack(outs).numpy(), world, 4 + 4 * B, need, need // 2)
            ref, gref = _reference_selection(f, a, y, C, ret, need, need // 2)
            ok &= bool(np.array_equal(picks, ref)) and abs(gap - gref) < 1e-15
        q.put((rank, bool(ok), ""))
    except Exception as e:
        q.put((rank, False, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def test_gloo_world2_intra_pair_candidate_merge():
    """NEXT-1's exchange: every rank's candidate block of its slice, all_gather over gloo, and the
    library's merge (gmpsvm_shard_merge) reproduces reading R19's selection on the whole vector
    (ties to the lowest index, I_u taken again when I_l runs short) and the global gap."""
    _run(_merge_worker, 2)
    _run(_merge_worker, 3)
