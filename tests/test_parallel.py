"""Multi-rank plumbing on CPU (gloo, world_size 2): slices, max-over-ranks,
stats gather.  The oracle stands in for the GPU solver (tests may call it);
the gathered per-system results must equal a single-process solve bitwise."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_kashinksla22_b200.parallel import gather_stats, max_over_ranks, rank_slice


def test_rank_slices_cover_exactly_once():
    for scaling in ("weak", "strong"):
        for world in (1, 2, 3, 8):
            for batch in (0, 1, 7, 100, 100_000):
                sl = [rank_slice(batch, r, world, scaling) for r in range(world)]
                idx = np.concatenate([np.arange(s.g0, s.g0 + s.count) for s in sl]) if batch else []
                total = batch * world if scaling == "weak" else batch
                assert len(idx) == total and all(s.total == total for s in sl)
                assert np.array_equal(idx, np.arange(total))
                if scaling == "strong" and batch:
                    c = [s.count for s in sl]
                    assert max(c) - min(c) <= 1


def test_rank_slice_errors():
    with pytest.raises(ValueError):
        rank_slice(10, 2, 2)
    with pytest.raises(ValueError):
        rank_slice(10, 0, 1, "diagonal")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, batch, scaling, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle as O
        import xgcgen as X
        sl = rank_slice(batch, rank, world, scaling)
        B = X.make_batch(sl.g0, sl.count)
        p = B.pattern
        o = O.batch_bicgstab(p.row_ptr, p.col_idx, B.values, B.b, threads=2)
        it, res, st = gather_stats(torch.from_numpy(o["iters"]), torch.from_numpy(o["resnorm"]),
                                   torch.from_numpy(o["status"].astype(np.int8)))
        t = max_over_ranks(float(rank + 1))
        if rank == 0:
            out.put((it.numpy(), res.numpy(), st.numpy(), t))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("scaling,batch", [("weak", 6), ("strong", 9)])
def test_gloo_world2_gather_matches_single_process(scaling, batch):
    import oracle as O
    import xgcgen as X
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, batch, scaling, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    it, res, st, t = q.get(timeout=300)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    total = batch * 2 if scaling == "weak" else batch
    B = X.make_batch(0, total)
    p = B.pattern
    o = O.batch_bicgstab(p.row_ptr, p.col_idx, B.values, B.b, threads=2)
    assert np.array_equal(it, o["iters"]) and np.array_equal(res, o["resnorm"])
    assert np.array_equal(st, o["status"].astype(np.int8))
    assert t == 2.0
