"""World-size-2 gloo test of the row-sharded SpMV host logic on CPU.

Each rank takes its nnz-balanced row range from the library's
dysel_partition_rows (host-only C ABI call), rebases row_ptr exactly as
bench.py / dysel_spmv_sharded do, computes its shard (with the fp64 oracle —
the device kernels need a GPU), and the shards are assembled with an
allgatherv over gloo.  The assembled y must equal the single-process oracle
bit for bit (same per-row order), proving partition + rebasing + assembly.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_main(rank, world, port, out_path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from oracle import spmv as ospmv
    from paper_conf_asplos_changkh16_b200 import dysel as D
    from workloads import d4_powerlaw, uniform_f32
    A = d4_powerlaw(n=30_000, lmax=3000)
    x = uniform_f32(77, A.n_cols)
    bounds = D.partition_rows(A.row_ptr, world)
    r0, r1 = bounds[rank], bounds[rank + 1]
    lo, hi = int(A.row_ptr[r0]), int(A.row_ptr[r1])
    rp_local = (A.row_ptr[r0:r1 + 1].astype(np.int64) - lo).astype(np.int32)
    y_local = ospmv.spmv(rp_local, A.col[lo:hi], A.val[lo:hi], x)
    # allgatherv: pad to the largest shard
    counts = [bounds[r + 1] - bounds[r] for r in range(world)]
    m = max(counts)
    buf = torch.zeros(m, dtype=torch.float64)
    buf[: len(y_local)] = torch.from_numpy(y_local)
    parts = [torch.zeros(m, dtype=torch.float64) for _ in range(world)]
    dist.all_gather(parts, buf)
    y = np.concatenate([parts[r][: counts[r]].numpy() for r in range(world)])
    if rank == 0:
        ref = ospmv.spmv(A.row_ptr, A.col, A.val, x)
        np.save(out_path, np.stack([y, ref]))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_row_sharded_spmv_assembles_exactly(tmp_path, world):
    out = str(tmp_path / "y.npy")
    mp.spawn(_rank_main, args=(world, _free_port(), out), nprocs=world, join=True)
    y, ref = np.load(out)
    assert np.array_equal(y, ref)


def test_allgather_chunks_tile_each_shard():
    """dysel_allgather_chunk (host C ABI): for any shard size the <= 8 chunks
    are whole 256-row units (the last may be ragged), disjoint, in order and
    cover [0, rows) exactly."""
    from paper_conf_asplos_changkh16_b200 import dysel as D
    for rows in (0, 1, 255, 256, 257, 2048, 2049, 300_000, 10_000_000, 123_457):
        ends = [D.allgather_chunk(rows, k) for k in range(8)]
        pos = 0
        for a, e in ends:
            assert a == min(pos, rows) and e >= a
            if e > a:
                assert a % 256 == 0 and (e % 256 == 0 or e == rows)
            pos = e if e > a else pos
        assert pos == rows, rows


def _rank_chunked(rank, world, port, out_path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from oracle import spmv as ospmv
    from paper_conf_asplos_changkh16_b200 import dysel as D
    from workloads import d4_powerlaw, uniform_f32
    A = d4_powerlaw(n=60_000, lmax=3000)
    x = uniform_f32(78, A.n_cols)
    bounds = D.partition_rows(A.row_ptr, world)
    r0, r1 = bounds[rank], bounds[rank + 1]
    lo, hi = int(A.row_ptr[r0]), int(A.row_ptr[r1])
    rp_local = (A.row_ptr[r0:r1 + 1].astype(np.int64) - lo).astype(np.int32)
    y = torch.zeros(A.n_rows, dtype=torch.float64)
    y[r0:r1] = torch.from_numpy(ospmv.spmv(rp_local, A.col[lo:hi], A.val[lo:hi], x))
    # the overlapped allgather's schedule (comm.cu): chunk k of every shard, root = its owner
    for k in range(8):
        for r in range(world):
            a, e = D.allgather_chunk(bounds[r + 1] - bounds[r], k)
            if e > a:
                part = y[bounds[r] + a: bounds[r] + e].clone()
                dist.broadcast(part, src=r)
                y[bounds[r] + a: bounds[r] + e] = part
    if rank == 1:
        ref = ospmv.spmv(A.row_ptr, A.col, A.val, x)
        np.save(out_path, np.stack([y.numpy(), ref]))
    dist.barrier()
    dist.destroy_process_group()


def test_chunked_allgather_schedule_world2(tmp_path):
    """World-2 gloo run of the overlapped allgather's chunk schedule: every
    rank derives every shard's chunks from bounds alone, so the per-chunk
    broadcasts match up and the assembled y (seen on rank 1) equals the
    single-process oracle bit for bit."""
    out = str(tmp_path / "y.npy")
    mp.spawn(_rank_chunked, args=(2, _free_port(), out), nprocs=2, join=True)
    y, ref = np.load(out)
    assert np.array_equal(y, ref)
