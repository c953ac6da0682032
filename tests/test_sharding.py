"""Multi-rank host logic on CPU with the gloo backend (world size 2 and 3).

Each rank regenerates its tensor range from the counter-based generator,
computes dedup records for it (the FP64 oracle stands in for the GPU solve on
this CPU-only box), packs them into the single int32 record buffer, and one
gather moves them to rank 0, which must reproduce the single-process result
for the whole volume bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_ballardkp11_b200 import sharding as SH
import synthetic as syn

M, N_DIM, S, KMAX = 4, 3, 16, 4
N_TOTAL = 10


def _records(first, count):
    from oracle import sshopm as O
    from oracle import dedup as D
    ent = syn.gen_voxels(M, N_DIM, first, count, seed=0)
    st = syn.gen_starts(S, N_DIM, seed=0)
    lam, x, it, cv = O.sshopm(ent, st, M, N_DIM, 0.0, 1e-6, 100)
    return D.dedup(lam.astype(np.float32), x.astype(np.float32), cv, M, 1e-2, 0.05, KMAX)


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    per = -(-N_TOTAL // world)                       # uniform per-rank size for the gather (padded)
    first, count = SH.shard_range(N_TOTAL, rank, world)
    buf = torch.zeros(SH.record_words(per, KMAX, N_DIM), dtype=torch.int32)
    views = SH.record_views(buf, per, KMAX, N_DIM)
    recs = _records(first, count)
    for v, r in zip(views, recs):
        v[:count] = torch.from_numpy(np.ascontiguousarray(r).astype(v.numpy().dtype))
    got = SH.gather_records(buf, rank, world)
    if rank == 0:
        parts = []
        for rk, b in enumerate(got):
            f, c = SH.shard_range(N_TOTAL, rk, world)
            parts.append(tuple(v[:c] for v in SH.record_views(b.numpy(), per, KMAX, N_DIM)))
        q.put(tuple(np.concatenate([p[i] for p in parts]) for i in range(5)))
    dist.barrier()
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_shard_range_partitions():
    for total in [0, 1, 7, 10, 1 << 20]:
        for world in [1, 2, 3, 8]:
            ranges = [SH.shard_range(total, r, world) for r in range(world)]
            assert ranges[0][0] == 0
            assert sum(c for _, c in ranges) == total
            for (f0, c0), (f1, _) in zip(ranges, ranges[1:]):
                assert f0 + c0 == f1
            assert max(c for _, c in ranges) - min(c for _, c in ranges) <= 1


def test_record_views_roundtrip():
    buf = np.zeros(SH.record_words(3, 2, 3), np.int32)
    c, lam, x, mu, rp = SH.record_views(buf, 3, 2, 3)
    lam[:] = [[1.5, -2.0], [0.25, 3.0], [7.0, 8.0]]
    x[1, 1] = [0.1, 0.2, 0.3]
    c[:] = [1, 2, 3]
    c2, lam2, x2, mu2, rp2 = SH.record_views(buf.copy(), 3, 2, 3)
    assert np.array_equal(lam2, lam) and np.array_equal(x2, x) and np.array_equal(c2, c)


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_gather_matches_single_process(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    merged = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    ref = _records(0, N_TOTAL)
    for a, b in zip(merged, ref):
        assert np.array_equal(np.asarray(a), np.asarray(b).astype(np.asarray(a).dtype))


def test_chunk_bounds_partition():
    for total in [0, 1, 5, 10, 1 << 20]:
        for c in [1, 2, 3, 4, 8]:
            b = SH.chunk_bounds(total, c)
            assert sum(v1 - v0 for v0, v1 in b) == total
            assert all(v1 > v0 for v0, v1 in b)
            for (a0, a1), (b0, _) in zip(b, b[1:]):
                assert a1 == b0
            if total:
                assert b[0][0] == 0 and len(b) == min(c, total)


def _chunked_worker(rank, world, chunks, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    per = N_TOTAL // world
    first, count = SH.shard_range(N_TOTAL, rank, world)
    words, _ = SH.chunked_record_words(per, chunks, KMAX, N_DIM)
    buf = torch.zeros(words, dtype=torch.int32)
    gathered = []
    for (v0, v1), (block, views) in zip(SH.chunk_bounds(per, chunks),
                                        SH.chunked_record_views(buf, per, chunks, KMAX, N_DIM)):
        recs = _records(first + v0, v1 - v0)          # chunk c is solved, deduped, then gathered on its own
        for v, r in zip(views, recs):
            v[:] = torch.from_numpy(np.ascontiguousarray(r).astype(v.numpy().dtype))
        gathered.append(SH.gather_records(block, rank, world))
    if rank == 0:
        q.put(SH.merge_chunked(gathered, per, chunks, KMAX, N_DIM))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_chunked_gather_matches_single_process():
    """Per-chunk gathers (the overlapped multi-GPU form) reassemble the whole volume bit for bit."""
    world, chunks = 2, 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_chunked_worker, args=(r, world, chunks, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    merged = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    ref = _records(0, N_TOTAL)
    for a, b in zip(merged, ref):
        assert np.array_equal(np.asarray(a), np.asarray(b).astype(np.asarray(a).dtype))
