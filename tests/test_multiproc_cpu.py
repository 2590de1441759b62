"""World-size-2 gloo tests of the multi-GPU path (pin P12).

CPU (no GPU here): ``multi.evaluate_distributed`` -- the product function -- runs on every rank of a
gloo group.  Rank 0 compresses (the oracle stands in for sg_hierarchize), the ONE broadcast replicates
the surpluses, every rank derives the same global order of the whole batch and evaluates its contiguous
range of it.  The grid object is a CPU stand-in whose ``sfc_order`` / ``evaluate_ordered`` follow the
C ABI's contract (sg_sfc_order: deterministic permutation of the whole batch; sg_evaluate_ordered:
y[perm[first+k]] for k < count) with the oracle as evaluator, so what is tested here is the
distribution logic: broadcast, agreement on one order, a partition that covers the batch exactly once,
and bitwise equality of the assembled shards with a single-process evaluation.  The same test with
libsg's kernels runs on one GPU in tests/test_gpu_parity.py (``-m gpu``).
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

D, N, M, SEED = 3, 5, 515, 0x5EED0099


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


class OracleGrid:
    """CPU stand-in with the Grid methods evaluate_distributed uses (sfc_order, evaluate_ordered)."""

    def __init__(self, d, n):
        import oracle
        self.oracle, self.d, self.n = oracle, d, n

    def sfc_order(self, x):
        # any deterministic function of the batch: lexicographic on the coordinates' finest cells
        cells = np.floor(x.numpy() * 1024).astype(np.int64)
        return torch.from_numpy(np.lexsort(cells.T[::-1]).astype(np.int32))

    def evaluate_ordered(self, alpha, x, perm, first, count, out=None):
        y = out if out is not None else torch.zeros(x.shape[0], dtype=x.dtype)
        idx = perm[first:first + count].long()
        yo, _ = self.oracle.evaluate(self.d, self.n, alpha.numpy(), x[idx].numpy())
        y[idx] = torch.from_numpy(np.ascontiguousarray(yo))
        return y


def _worker(rank, world, port, outdir):
    import oracle
    import sginputs as S
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = OracleGrid(D, N)
        alpha = torch.zeros(oracle.num_points(D, N), dtype=torch.float64)
        if rank == 0:  # compression on rank 0 only
            alpha.copy_(torch.from_numpy(oracle.hierarchize(D, N, S.f_A(oracle.coords(D, N)))))
        x = torch.from_numpy(S.queries(D, M, SEED))  # the whole batch, on every rank
        y, perm, first, count = multi.evaluate_distributed(g, alpha, x)
        c = multi.checksum(alpha)
        meta = torch.tensor([c - (1 << 64) if c >= (1 << 63) else c, first, count, multi.checksum(perm) >> 1],
                            dtype=torch.int64)
        # test-side verification only: collect every rank's shard and metadata on rank 0
        metas = [torch.zeros_like(meta) for _ in range(world)]
        ys = [torch.zeros_like(y) for _ in range(world)]
        dist.all_gather(metas, meta)
        dist.all_gather(ys, y)
        if rank == 0:
            np.save(os.path.join(outdir, "meta.npy"), torch.stack(metas).numpy())
            np.save(os.path.join(outdir, "ys.npy"), torch.stack(ys).numpy())
            np.save(os.path.join(outdir, "perm.npy"), perm.numpy())
            np.save(os.path.join(outdir, "alpha.npy"), alpha.numpy())
    finally:
        dist.destroy_process_group()


def test_partition_covers_the_order_exactly_once():
    from paper_conf_ppopp_murarasuwbbp11_b200 import multi
    for m in (0, 1, 7, 8, 10_000_000, 10_000_003):
        for world in (1, 2, 3, 4, 8):
            ranges = [multi.partition(m, world, r) for r in range(world)]
            assert ranges[0][0] == 0 and sum(c for _, c in ranges) == m
            assert all(f0 + c0 == f1 for (f0, c0), (f1, _) in zip(ranges, ranges[1:]))
            assert max(c for _, c in ranges) - min(c for _, c in ranges) <= 1  # static balance
    with pytest.raises(ValueError):
        multi.partition(5, 2, 2)
    with pytest.raises(ValueError):
        multi.partition(-1, 1, 0)


def test_gloo_world2_evaluate_distributed(tmp_path, oracle):
    import sginputs as S
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    meta = np.load(tmp_path / "meta.npy")
    ys = np.load(tmp_path / "ys.npy")
    perm = np.load(tmp_path / "perm.npy")
    alpha = np.load(tmp_path / "alpha.npy")
    assert len(set(meta[:, 0].tolist())) == 1  # every rank holds the same surplus bytes (one broadcast)
    assert len(set(meta[:, 3].tolist())) == 1  # every rank derived the same global order
    assert sorted(perm.tolist()) == list(range(M))
    # the ranks' ranges tile the order; each rank wrote exactly its queries
    assert meta[0, 1] == 0 and meta[0, 2] + meta[1, 2] == M and meta[1, 1] == meta[0, 2]
    x_all = S.queries(D, M, SEED)
    y_ref, _ = oracle.evaluate(D, N, alpha, x_all)
    assembled = np.zeros(M)
    for r in range(world):
        own = perm[meta[r, 1]:meta[r, 1] + meta[r, 2]]
        others = np.setdiff1d(np.arange(M), own)
        assert np.all(ys[r][others] == 0.0)
        assembled[own] = ys[r][own]
    assert np.array_equal(assembled, y_ref)  # bitwise: shards == one process, whole batch
    assert np.array_equal(alpha, oracle.hierarchize(D, N, S.f_A(oracle.coords(D, N))))
