"""The multi-GPU driver with several real processes (PAPER.md L311 pairs are
independent, L273 test instances are independent): world_size 2 and 4 over gloo, every rank on
cuda:0 (only one GPU per call here; the NCCL path differs only in the backend).  Each rank trains
its LPT shard of pairs (pair_ids), the disjoint solutions are all-reduced, every rank rebuilds the
complete model (gmpsvm_model_from_alpha) and predicts its row shard; the all-gathered
probabilities must be BITWISE those of one process training every pair.  k = 3 on 4 ranks leaves
one rank without a pair (it trains nothing and contributes zeros).  The intra-pair sharded solver
(NEXT-1, dist.train_pair_sharded) is checked the same way in test_gpu_shard.py."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, name, n, m, q):
    try:
        import sys

        sys.path.insert(0, ROOT)
        import torch.distributed as dist

        import datagen
        from paper_conf_icde_wenshcc19_b200 import dist as gdist

        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=m)
        Xd, yd, Xtd = (torch.from_numpy(a).cuda() for a in (X, y, Xt))
        model, prob = gdist.train_predict(Xd, yd, Xtd, spec.k, spec.C, spec.gamma, 1e-5)
        q.put((rank, prob.cpu().numpy(), model.sv_index(), model.n_sv, ""))
    except Exception as e:  # report instead of hanging the parent
        q.put((rank, None, None, None, repr(e)))
    finally:
        import torch.distributed as dist

        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("name,n,m,world", [("mnist", 2000, 300, 2), ("blobs", None, None, 4), ("letter", 2600, 200, 2)])
def test_multiprocess_train_predict_bitwise(name, n, m, world):
    import torch.multiprocessing as mp

    import __graft_entry__
    import datagen

    __graft_entry__.build()
    import paper_conf_icde_wenshcc19_b200 as gm

    spec, X, y, Xt, yt = datagen.make_config(name, n_train=n, n_test=m)
    full = gm.train(X, y, spec.k, spec.C, spec.gamma, 1e-5)
    p_full = full.predict_proba(Xt)
    ctx = mp.get_context("spawn")
    qu = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, n, m, qu)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([qu.get(timeout=600) for _ in procs], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
    assert all(r[4] == "" for r in res), [r[4] for r in res]
    for rank, prob, svi, nsv, _ in res:
        np.testing.assert_array_equal(prob, p_full)
        assert nsv == full.n_sv
        np.testing.assert_array_equal(svi, full.sv_index())
