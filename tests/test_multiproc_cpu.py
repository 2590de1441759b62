"""World-size-2 gloo tests of the multi-GPU host logic (pin P12).

Runs on CPU: rank 0 compresses (the oracle stands in for sg_hierarchize, since
there is no GPU here), ONE broadcast replicates the surpluses
(multi.replicate_surpluses, the path's only collective), every rank evaluates
its shard of the global query stream (multi.shard_range), and rank 0 checks
that the gathered shards are bitwise identical to a single-process evaluation
of the whole batch (partition invariance) and that every rank holds the same
surplus bytes (broadcast checksum).
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

D, N, M_PER_RANK, SEED = 3, 5, 257, 0x5EED0099


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, outdir):
    import oracle
    import sginputs as S
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        npts = oracle.num_points(D, N)
        alpha = torch.zeros(npts, dtype=torch.float64)
        if rank == 0:  # compression on rank 0 only
            coords = oracle.coords(D, N)
            alpha.copy_(torch.from_numpy(oracle.hierarchize(D, N, S.f_A(coords))))
        multi.replicate_surpluses(alpha, src=0)
        c = multi.checksum(alpha)
        cs = torch.tensor([c - (1 << 64) if c >= (1 << 63) else c], dtype=torch.int64)
        all_cs = [torch.zeros_like(cs) for _ in range(world)]
        dist.all_gather(all_cs, cs)  # test-side verification only
        first, count = multi.shard_range(M_PER_RANK, rank)
        x = S.queries(D, count, SEED, first=first)
        y, _ = oracle.evaluate(D, N, alpha.numpy(), x)
        yt = torch.from_numpy(np.ascontiguousarray(y))
        gathered = [torch.zeros_like(yt) for _ in range(world)] if rank == 0 else None
        dist.gather(yt, gathered, dst=0)
        if rank == 0:
            np.save(os.path.join(outdir, "y.npy"), torch.cat(gathered).numpy())
            np.save(os.path.join(outdir, "cs.npy"), torch.cat(all_cs).numpy())
            np.save(os.path.join(outdir, "alpha.npy"), alpha.numpy())
    finally:
        dist.destroy_process_group()


def test_shard_range_partitions_the_stream():
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi
    rows = [multi.shard_range(7, r) for r in range(4)]
    assert rows == [(0, 7), (7, 7), (14, 7), (21, 7)]
    import sginputs as S
    whole = S.queries(3, 28, SEED)
    parts = np.concatenate([S.queries(3, c, SEED, first=f) for f, c in rows])
    assert np.array_equal(whole, parts)
    with pytest.raises(ValueError):
        multi.shard_range(-1, 0)


def test_gloo_world2_broadcast_and_partition_invariance(tmp_path, oracle):
    import sginputs as S
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    y = np.load(tmp_path / "y.npy")
    cs = np.load(tmp_path / "cs.npy")
    alpha = np.load(tmp_path / "alpha.npy")
    # every rank holds the same surplus bytes after the one broadcast
    assert len(set(cs.tolist())) == 1
    # gathered shards == one process evaluating the whole global batch, bitwise
    x_all = S.queries(D, world * M_PER_RANK, SEED)
    y_ref, _ = oracle.evaluate(D, N, alpha, x_all)
    assert np.array_equal(y, y_ref)
    # and the broadcast payload is rank 0's compression of f_A
    a_ref = oracle.hierarchize(D, N, S.f_A(oracle.coords(D, N)))
    assert np.array_equal(alpha, a_ref)
