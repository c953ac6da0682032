"""CPU-side checks of the C-ABI library (no GPU needed).

* the shared library loads and exports every function include/sshopm.h declares;
* host-only entry points (create / num_unique / class_index / flops / errors)
  behave as documented;
* the library's compile-time class enumeration equals the oracle's
  independent enumeration (T0 in SURVEY.md Sec. 4).
"""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_ballardkp11_b200 as sh
from oracle import sshopm as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    with open(os.path.join(ROOT, "include", "sshopm.h")) as f:
        txt = f.read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(sshopm_[a-z_]+)\s*\(", txt)))


def test_library_exports_header_symbols():
    L = sh.lib()
    names = _header_functions()
    assert len(names) >= 14
    for name in names:
        assert hasattr(L, name), name


def test_create_errors():
    L = sh.lib()
    h = ctypes.c_void_p()
    assert L.sshopm_create(1, 3, ctypes.byref(h)) == sh.EINVAL
    assert L.sshopm_create(4, 0, ctypes.byref(h)) == sh.EINVAL
    assert L.sshopm_create(4, 3, None) == sh.EINVAL
    assert L.sshopm_create(17, 3, ctypes.byref(h)) == sh.EUNSUPPORTED      # beyond the general kernel's m <= 16
    assert L.sshopm_create(4, 17, ctypes.byref(h)) == sh.EUNSUPPORTED
    assert L.sshopm_destroy(None) == sh.OK
    with pytest.raises(sh.SSHOPMError):
        sh.Solver(20, 20)


def test_status_strings():
    L = sh.lib()
    for c in range(5):
        assert len(L.sshopm_status_string(c)) > 0


@pytest.mark.parametrize("m,n", sh.supported_shapes() if os.path.exists(sh.library_path) else [])
def test_class_index_matches_oracle_enumeration(m, n):
    s = sh.Solver(m, n)
    assert s.U == O.num_unique(m, n)
    assert np.array_equal(s.class_index(), np.array(O.class_list(m, n), dtype=np.int32))
    assert s.paper_flops_per_iter == O.paper_flops_per_iter(m, n)
    assert s.exec_flops_per_iter > 0
    s.close()


def test_required_shapes_compiled():
    shapes = set(sh.supported_shapes())
    for need in [(4, 3), (6, 3), (8, 3), (4, 6), (2, 3)]:
        assert need in shapes


def test_host_side_argument_validation():
    """Synchronous checks return EINVAL before touching the device."""
    L = sh.lib()
    s = sh.Solver(4, 3)
    P = ctypes.c_void_p
    # N = 0 is a no-op
    assert L.sshopm_solve(s._h, 0, None, 128, None, 0.0, 1e-6, 100, None, None, None, None, None) == sh.OK
    # null pointers with N > 0, bad S / maxit / NaN
    assert L.sshopm_solve(s._h, 10, None, 128, None, 0.0, 1e-6, 100, None, None, None, None, None) == sh.EINVAL
    dummy = P(16)
    args = (dummy, dummy, dummy, dummy)
    assert L.sshopm_solve(s._h, 10, dummy, 0, dummy, 0.0, 1e-6, 100, *args, None) == sh.EINVAL
    assert L.sshopm_solve(s._h, 10, dummy, 8, dummy, 0.0, 1e-6, -1, *args, None) == sh.EINVAL
    assert L.sshopm_solve(s._h, 10, dummy, 8, dummy, float("nan"), 1e-6, 10, *args, None) == sh.EINVAL
    assert L.sshopm_solve(None, 10, dummy, 8, dummy, 0.0, 1e-6, 10, *args, None) == sh.EINVAL
    # dedup: kmax < 1, negative / NaN tolerances, S too large
    d5 = (dummy,) * 5
    assert L.sshopm_dedup(s._h, 10, 8, dummy, dummy, dummy, 0.01, 0.05, 0, *d5, None) == sh.EINVAL
    assert L.sshopm_dedup(s._h, 10, 8, dummy, dummy, dummy, -1.0, 0.05, 4, *d5, None) == sh.EINVAL
    assert L.sshopm_dedup(s._h, 10, 8, dummy, dummy, dummy, 0.01, float("nan"), 4, *d5, None) == sh.EINVAL
    assert L.sshopm_dedup(s._h, 10, 2048, dummy, dummy, dummy, 0.01, 0.05, 4, *d5, None) == sh.EUNSUPPORTED
    assert L.sshopm_apply(s._h, 0, None, None, None, None, None) == sh.OK
    assert L.sshopm_apply(s._h, 3, None, None, None, None, None) == sh.EINVAL
    s.close()


@pytest.mark.parametrize("m,n", [(5, 4), (7, 2), (3, 6), (9, 3), (2, 9), (6, 5), (10, 2)])
def test_general_shapes_tables(m, n):
    """(m, n) without a compiled kernel: the general kernel's Fig. 4 tables equal the oracle's enumeration."""
    assert (m, n) not in set(sh.supported_shapes())
    s = sh.Solver(m, n)
    assert s.U == O.num_unique(m, n)
    assert np.array_equal(s.class_index(), np.array(O.class_list(m, n), dtype=np.int32))
    assert s.paper_flops_per_iter == O.paper_flops_per_iter(m, n)
    s.close()


def test_ipc_entry_points_reject_bad_arguments():
    """Peer-memory gather entry points (multi-GPU A9): argument checks happen before any CUDA call."""
    L = sh.lib()
    p = ctypes.c_void_p()
    h = ctypes.create_string_buffer(sh.IPC_HANDLE_BYTES)
    assert L.sshopm_ipc_alloc(0, ctypes.byref(p), h) == sh.EINVAL
    assert L.sshopm_ipc_alloc(1024, None, h) == sh.EINVAL
    assert L.sshopm_ipc_alloc(1024, ctypes.byref(p), None) == sh.EINVAL
    assert L.sshopm_ipc_import(None, ctypes.byref(p)) == sh.EINVAL
    assert L.sshopm_ipc_import(h, None) == sh.EINVAL
    assert L.sshopm_ipc_free(None) == sh.EINVAL
    assert L.sshopm_ipc_release(None) == sh.EINVAL
