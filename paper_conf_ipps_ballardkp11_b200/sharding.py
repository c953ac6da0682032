"""Multi-GPU host logic: tensor-range sharding and the dedup-record gather.

The path partitions (independent tensors; "generalizes to a system
with multiple GPUs"): rank r of P owns a contiguous range of tensors,
solves and dedups it locally, and one collective moves the fixed-size
per-tensor dedup records to rank 0.  No data-path
collective exists during the solve.

Overlap: a rank may split its range into C contiguous chunks
(`chunk_bounds`) with one record block per chunk (`chunked_record_views`);
chunk i's block is gathered on a side stream while chunk i+1 solves, so only
the last chunk's gather is exposed.  `merge_chunked` reassembles rank 0's
gathered blocks in global tensor order.

Record layout (one int32 buffer per rank, so a single collective moves it):
    count [N] i32 | lambda [N, K] f32 | x [N, K, n] f32 | mult [N, K] i32 | rep [N, K] i32
Float fields are stored bit-for-bit (reinterpreted as int32).  All ranks use
the same per-rank N (weak scaling) so the gather is uniform.
"""
import numpy as np


def shard_range(n_total, rank, world):
    """[first, first+count) of the tensors owned by `rank` (contiguous, balanced, covers n_total)."""
    base, extra = divmod(int(n_total), int(world))
    first = rank * base + min(rank, extra)
    return first, base + (1 if rank < extra else 0)


def record_words(n_tensors, kmax, n):
    return n_tensors * (1 + kmax * (n + 3))


def record_views(buf, n_tensors, kmax, n):
    """Split a flat int32 torch/numpy buffer into (count, lambda, x, mult, rep) views (no copies)."""
    shapes = [((n_tensors,), "i"), ((n_tensors, kmax), "f"), ((n_tensors, kmax, n), "f"),
              ((n_tensors, kmax), "i"), ((n_tensors, kmax), "i")]
    out, o = [], 0
    for shape, kind in shapes:
        cnt = int(np.prod(shape))
        seg = buf[o:o + cnt]
        if kind == "f":
            seg = seg.view(np.float32) if isinstance(seg, np.ndarray) else seg.view(_torch().float32)
        out.append(seg.reshape(shape) if isinstance(seg, np.ndarray) else seg.view(shape))
        o += cnt
    return tuple(out)


def _torch():
    import torch
    return torch


def gather_records(rec, rank, world, group=None):
    """Gather every rank's record buffer to rank 0 (one collective).  Returns the list on rank 0, else None."""
    import torch.distributed as dist
    if world == 1:
        return [rec]
    out = [rec.new_empty(rec.shape) for _ in range(world)] if rank == 0 else None
    dist.gather(rec, out, dst=0, group=group)
    return out


def merge_records(bufs, n_per_rank, kmax, n, n_total=None):
    """Rank-0 side: concatenate gathered buffers into global (count, lambda, x, mult, rep) host arrays."""
    parts = [record_views(b.cpu().numpy() if hasattr(b, "cpu") else b, n_per_rank, kmax, n) for b in bufs]
    merged = tuple(np.concatenate([p[i] for p in parts], axis=0) for i in range(5))
    if n_total is not None:
        merged = tuple(m[:n_total] for m in merged)
    return merged


def chunk_bounds(n_tensors, n_chunks):
    """[(v0, v1)] of `n_chunks` contiguous, balanced sub-ranges covering [0, n_tensors) (empty ones dropped)."""
    n_chunks = max(1, min(int(n_chunks), max(1, int(n_tensors))))
    out = []
    for c in range(n_chunks):
        f, k = shard_range(n_tensors, c, n_chunks)
        if k > 0:
            out.append((f, f + k))
    return out


def chunked_record_words(n_tensors, n_chunks, kmax, n):
    """Words of a buffer holding one record block per chunk, each sized for the largest chunk
    (identical on every rank because all ranks hold the same number of tensors)."""
    bounds = chunk_bounds(n_tensors, n_chunks)
    per = max((v1 - v0 for v0, v1 in bounds), default=0)
    return len(bounds) * record_words(per, kmax, n), per


def chunked_record_views(buf, n_tensors, n_chunks, kmax, n):
    """[(block, views)] per chunk: `block` is the chunk's flat slice of `buf` (what one gather moves),
    `views` its (count, lambda, x, mult, rep) fields sized for the chunk's own tensor count."""
    bounds = chunk_bounds(n_tensors, n_chunks)
    _, per = chunked_record_words(n_tensors, n_chunks, kmax, n)
    w = record_words(per, kmax, n)
    out = []
    for i, (v0, v1) in enumerate(bounds):
        block = buf[i * w:(i + 1) * w]
        views = tuple(v[:v1 - v0] for v in record_views(block, per, kmax, n))
        out.append((block, views))
    return out


def merge_chunked(gathered, n_per_rank, n_chunks, kmax, n):
    """Rank-0 side: gathered[c][r] = rank r's block of chunk c (from one gather per chunk).
    Returns global (count, lambda, x, mult, rep) host arrays in tensor order (rank-major, then chunk)."""
    bounds = chunk_bounds(n_per_rank, n_chunks)
    _, per = chunked_record_words(n_per_rank, n_chunks, kmax, n)
    world = len(gathered[0])
    parts = []
    for r in range(world):
        for c, (v0, v1) in enumerate(bounds):
            b = gathered[c][r]
            b = b.cpu().numpy() if hasattr(b, "cpu") else np.asarray(b)
            parts.append(tuple(v[:v1 - v0] for v in record_views(b, per, kmax, n)))
    return tuple(np.concatenate([p[i] for p in parts], axis=0) for i in range(5))


class PeerRecords:
    """Rank 0's gather buffer, mapped into every rank through the library's IPC entry points
    (sshopm_ipc_alloc / sshopm_ipc_import): rank r passes views of its own slice as sshopm_dedup's
    outputs, so the dedup kernel stores its records over NVLink straight into rank 0's memory — the
    gather is fused into the producing kernel.  Layout: [world][chunked record
    buffer of one rank] (chunked_record_words), so merge_chunked reassembles it like gathered blocks."""

    def __init__(self, n_per_rank, n_chunks, kmax, n, rank, world, device):
        import torch
        import torch.distributed as dist
        import paper_conf_ipps_ballardkp11_b200 as sh
        self.rank, self.world, self.n_chunks, self.kmax, self.n = rank, world, n_chunks, kmax, n
        self.n_per_rank = n_per_rank
        self.words, _ = chunked_record_words(n_per_rank, n_chunks, kmax, n)
        obj = [None]
        if rank == 0:
            self.ptr, handle = sh.ipc_alloc(4 * self.words * world)
            obj = [handle]
        if world > 1:
            dist.broadcast_object_list(obj, src=0)
        if rank != 0:
            self.ptr = sh.ipc_import(obj[0])
        self.buf = sh.device_view(self.ptr, (world * self.words,), torch.int32, device)
        self.slices = [self.buf[r * self.words:(r + 1) * self.words] for r in range(world)]
        self.blocks = chunked_record_views(self.slices[rank], n_per_rank, n_chunks, kmax, n)

    def merged(self):
        """Rank 0, after every rank's kernels finished (barrier): global records in tensor order."""
        gathered = [[chunked_record_views(self.slices[r], self.n_per_rank, self.n_chunks, self.kmax, self.n)[c][0]
                     for r in range(self.world)] for c in range(len(self.blocks))]
        return merge_chunked(gathered, self.n_per_rank, self.n_chunks, self.kmax, self.n)

    def close(self):
        import paper_conf_ipps_ballardkp11_b200 as sh
        self.buf = self.slices = self.blocks = None
        if self.rank == 0:
            sh.ipc_free(self.ptr)
        else:
            sh.ipc_release(self.ptr)
