"""64-bit item indexing (N*S >= 2^31): the WIDE kernels must give bit-identical per-lane results.

2^24 + 1024 tensors x 128 starts (~45 GB of raw outputs on a 180 GB B200).  The
entries tile one 2^20-tensor base set, so every tile must equal the 32-bit
path's results for the base set bit for bit (per-lane arithmetic does not
depend on scheduling or index width)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_ballardkp11_b200 as sh  # noqa: E402
import synthetic as syn  # noqa: E402


def test_wide_index_path_bitwise():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    free, _ = torch.cuda.mem_get_info()
    if free < 60e9:
        pytest.skip("needs ~60 GB of device memory")
    dev = torch.device("cuda:0")
    m, n, S = 4, 3, 128
    B = 1 << 20
    N = (1 << 24) + 1024
    assert N * S >= (1 << 31)
    base = torch.from_numpy(syn.gen_voxels(m, n, 0, B, 0)).to(dev)
    st = torch.from_numpy(syn.gen_starts(S, n, 0)).to(dev)
    s = sh.Solver(m, n)
    ref = s.solve(base, st, 0.0, 1e-6, 100)                          # 32-bit index path
    ent = base.repeat((N + B - 1) // B, 1)[:N].contiguous()
    out = s.solve(ent, st, 0.0, 1e-6, 100)                           # 64-bit index path
    torch.cuda.synchronize()
    for r, o in zip(ref, out):
        for t in range(N // B):
            assert torch.equal(o[t * B:(t + 1) * B], r), t
        tail = N - (N // B) * B
        assert torch.equal(o[(N // B) * B:], r[:tail])
    del out, ent
    torch.cuda.empty_cache()
