"""Multi-GPU host logic: tensor-range sharding and the dedup-record gather.

The path partitions (independent tensors; "generalizes to a system
with multiple GPUs"): rank r of P owns a contiguous range of tensors,
solves and dedups it locally, and one collective moves the fixed-size
per-tensor dedup records to rank 0.  No data-path
collective exists during the solve.

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
