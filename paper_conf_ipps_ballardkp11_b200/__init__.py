"""Batched SS-HOPM on B200 — thin Python binding over libsshopm.so (include/sshopm.h).

Argument marshalling only: every step of the hot path runs in the CUDA
kernels of the C-ABI library.  PyTorch provides device memory and streams.
There is no CPU fallback: if the library is missing, every call raises.

    import paper_conf_ipps_ballardkp11_b200 as sh
    solver = sh.Solver(4, 3)
    lam, x, iters, conv = solver.solve(entries, starts, alpha=0.0, tol=1e-6, maxit=100)
    count, clam, cx, mult, rep = solver.dedup(lam, x, conv)
"""
import ctypes
import os

import numpy as np

__all__ = ["Solver", "SSHOPMError", "lib", "supported_shapes", "library_path"]

_HERE = os.path.dirname(os.path.abspath(__file__))
# SSHOPM_LIBRARY: load a variant build (tools/ sweeps) instead of the in-tree product library
library_path = os.environ.get("SSHOPM_LIBRARY") or os.path.join(_HERE, "_lib", "libsshopm.so")
_LIB = None

OK, EINVAL, EUNSUPPORTED, ECUDA, ENOMEM = 0, 1, 2, 3, 4


class SSHOPMError(RuntimeError):
    def __init__(self, code, where):
        msg = f"{where}: status {code} ({_status(code)})"
        if code == ECUDA:
            msg += ": " + lib().sshopm_last_cuda_error().decode()
        super().__init__(msg)
        self.code = code


class _Opts(ctypes.Structure):
    _fields_ = [("refill_threshold", ctypes.c_int), ("ctas_per_sm", ctypes.c_int),
                ("d_total_iters", ctypes.c_void_p), ("d_workspace", ctypes.c_void_p),
                ("workspace_bytes", ctypes.c_size_t), ("schedule", ctypes.c_int), ("fuse_dedup", ctypes.c_int),
                ("alpha_mode", ctypes.c_int), ("d_alpha", ctypes.c_void_p), ("chunk_tensors", ctypes.c_int),
                ("d_records", ctypes.c_void_p), ("records_bytes", ctypes.c_size_t), ("unit_starts", ctypes.c_int)]

ALPHA_MODES = {"scalar": 0, "per_tensor": 1, "auto_max": 2, "auto_min": 3}


def lib():
    """Load libsshopm.so (built by __graft_entry__.build()); raises if absent."""
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(library_path):
        raise RuntimeError(f"{library_path} is not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(library_path)
    P, I, I64, F = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_float
    sig = {
        "sshopm_create": (I, [I, I, ctypes.POINTER(P)]),
        "sshopm_destroy": (I, [P]),
        "sshopm_num_unique": (I, [P, ctypes.POINTER(I)]),
        "sshopm_class_index": (I, [P, P]),
        "sshopm_flops_per_iter": (I, [P, ctypes.POINTER(I64), ctypes.POINTER(I64)]),
        "sshopm_solve": (I, [P, I64, P, I, P, F, F, I, P, P, P, P, P]),
        "sshopm_solve_ex": (I, [P, I64, P, I, P, F, F, I, P, P, P, P, ctypes.POINTER(_Opts), P]),
        "sshopm_dedup": (I, [P, I64, I, P, P, P, F, F, I, P, P, P, P, P, P]),
        "sshopm_solve_dedup": (I, [P, I64, P, I, P, F, F, I, P, P, P, P, F, F, I, P, P, P, P, P,
                                   ctypes.POINTER(_Opts), P]),
        "sshopm_apply": (I, [P, I64, P, P, P, P, P]),
        "sshopm_classify": (I, [P, I64, P, I, P, P, P, F, P, P]),
        "sshopm_run_host": (I, [P, I64, P, I, P, F, F, I, F, F, I, P, P, P, P, P, P, P, P, P, I64, P]),
        "sshopm_launch_count": (I, [P, ctypes.POINTER(I64)]),
        "sshopm_workspace_size": (I, [P, I64, I, ctypes.POINTER(ctypes.c_size_t)]),
        "sshopm_records_size": (I, [P, I64, I, ctypes.POINTER(ctypes.c_size_t)]),
        "sshopm_status_string": (ctypes.c_char_p, [I]),
        "sshopm_last_cuda_error": (ctypes.c_char_p, []),
        "sshopm_supported_shapes": (ctypes.c_char_p, []),
        "sshopm_ipc_alloc": (I, [ctypes.c_size_t, ctypes.POINTER(P), P]),
        "sshopm_ipc_free": (I, [P]),
        "sshopm_ipc_import": (I, [P, ctypes.POINTER(P)]),
        "sshopm_ipc_release": (I, [P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _LIB = L
    return L


def _status(code):
    return lib().sshopm_status_string(code).decode()


def _check(code, where):
    if code != OK:
        raise SSHOPMError(code, where)


IPC_HANDLE_BYTES = 64


def ipc_alloc(nbytes):
    """Device buffer other processes of this node can map: -> (device address, handle bytes)."""
    p = ctypes.c_void_p()
    h = ctypes.create_string_buffer(IPC_HANDLE_BYTES)
    _check(lib().sshopm_ipc_alloc(ctypes.c_size_t(int(nbytes)), ctypes.byref(p), h), "sshopm_ipc_alloc")
    return int(p.value), h.raw


def ipc_free(ptr):
    _check(lib().sshopm_ipc_free(ctypes.c_void_p(ptr)), "sshopm_ipc_free")


def ipc_import(handle):
    """Map another process's exported allocation; returns its device address (int)."""
    p = ctypes.c_void_p()
    _check(lib().sshopm_ipc_import(ctypes.create_string_buffer(bytes(handle), IPC_HANDLE_BYTES), ctypes.byref(p)),
           "sshopm_ipc_import")
    return int(p.value)


def ipc_release(ptr):
    _check(lib().sshopm_ipc_release(ctypes.c_void_p(ptr)), "sshopm_ipc_release")


class _CudaArray:
    """__cuda_array_interface__ wrapper: lets torch alias a raw device address without a copy."""

    def __init__(self, ptr, shape, typestr):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def device_view(ptr, shape, dtype, device):
    """A torch tensor aliasing `ptr` (e.g. a peer buffer mapped by ipc_import); no copy."""
    torch = _torch()
    ts = {torch.int32: "<i4", torch.float32: "<f4", torch.uint8: "|u1"}[dtype]
    return torch.as_tensor(_CudaArray(ptr, shape, ts), device=device)


def supported_shapes():
    """[(m, n), ...] compiled into the library."""
    s = lib().sshopm_supported_shapes().decode()
    return [tuple(int(t) for t in p.split("x")) for p in s.split(",") if p]


def _torch():
    import torch
    return torch


def _dev(t, dtype, shape, name):
    torch = _torch()
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA torch.Tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} must have shape {tuple(shape)}, got {tuple(t.shape)}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return ctypes.c_void_p(t.data_ptr())


def _stream(stream):
    torch = _torch()
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


class Solver:
    """Handle for tensors of order m, dimension n (sshopm_create)."""

    def __init__(self, m, n):
        h = ctypes.c_void_p()
        _check(lib().sshopm_create(int(m), int(n), ctypes.byref(h)), f"sshopm_create({m},{n})")
        self._h = h
        self.m, self.n = int(m), int(n)
        u = ctypes.c_int()
        _check(lib().sshopm_num_unique(h, ctypes.byref(u)), "sshopm_num_unique")
        self.U = u.value
        pf, ef = ctypes.c_int64(), ctypes.c_int64()
        _check(lib().sshopm_flops_per_iter(h, ctypes.byref(pf), ctypes.byref(ef)), "sshopm_flops_per_iter")
        self.paper_flops_per_iter = pf.value
        self.exec_flops_per_iter = ef.value
        self._ws = {}              # (device, stream handle) -> cached device workspace (torch uint8 tensor)
        self._ws_size = {}         # (N, S) -> bytes

    def close(self):
        if getattr(self, "_h", None):
            lib().sshopm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def class_index(self):
        out = np.zeros((self.U, self.m), dtype=np.int32)
        _check(lib().sshopm_class_index(self._h, out.ctypes.data_as(ctypes.c_void_p)), "sshopm_class_index")
        return out

    def workspace_size(self, N, S):
        key = (int(N), int(S))
        if key not in self._ws_size:
            b = ctypes.c_size_t()
            _check(lib().sshopm_workspace_size(self._h, int(N), int(S), ctypes.byref(b)), "sshopm_workspace_size")
            self._ws_size[key] = b.value
        return self._ws_size[key]

    def _workspace(self, N, S, device, stream=None):
        """Workspace for a call on `stream`: one cached buffer per (device, stream), allocated on that
        stream, so calls in flight on different streams never share (or free) each other's workspace."""
        need = self.workspace_size(N, S)
        torch = _torch()
        st = torch.cuda.current_stream(device) if stream is None else stream
        key = (str(device), int(st.cuda_stream))
        ws = self._ws.get(key)
        if ws is None or ws.numel() < need:
            with torch.cuda.stream(st):
                ws = torch.empty(need + 256, dtype=torch.uint8, device=device)
            old = self._ws.get(key)
            if old is not None:
                old.record_stream(st)      # the previous buffer stays alive until the stream's queued work ends
            self._ws[key] = ws
        base = ws.data_ptr()
        return ctypes.c_void_p((base + 255) // 256 * 256), need

    def _records(self, N, S, device, stream=None):
        """Record scratch of the records path (fuse_dedup = 4), cached per (device, stream) like the workspace."""
        b = ctypes.c_size_t()
        _check(lib().sshopm_records_size(self._h, int(N), int(S), ctypes.byref(b)), "sshopm_records_size")
        need = int(b.value)
        torch = _torch()
        st = torch.cuda.current_stream(device) if stream is None else stream
        key = ("rec", str(device), int(st.cuda_stream))
        buf = self._ws.get(key)
        if buf is None or buf.numel() < need:
            with torch.cuda.stream(st):
                buf = torch.empty(need + 256, dtype=torch.uint8, device=device)
            old = self._ws.get(key)
            if old is not None:
                old.record_stream(st)
            self._ws[key] = buf
        base = buf.data_ptr()
        return ctypes.c_void_p((base + 255) // 256 * 256), need

    @staticmethod
    def _alpha_opts(alpha, N, opts):
        """alpha: float (scalar shift), a CUDA float32 tensor [N] (per tensor), or 'auto_max' / 'auto_min'."""
        if isinstance(alpha, str):
            if alpha not in ("auto_max", "auto_min"):
                raise ValueError("alpha must be a float, a [N] tensor, 'auto_max' or 'auto_min'")
            opts.alpha_mode = ALPHA_MODES[alpha]
            return 0.0
        if hasattr(alpha, "data_ptr"):
            torch = _torch()
            _dev(alpha, torch.float32, (N,), "alpha")
            opts.alpha_mode = 1
            opts.d_alpha = alpha.data_ptr()
            return 0.0
        return float(alpha)

    def launch_count(self):
        c = ctypes.c_int64()
        _check(lib().sshopm_launch_count(self._h, ctypes.byref(c)), "sshopm_launch_count")
        return c.value

    def solve(self, entries, starts, alpha=0.0, tol=1e-6, maxit=100, out=None, refill_threshold=0,
              ctas_per_sm=0, total_iters=None, stream=None, schedule=0, chunk_tensors=0):
        """entries [N, U] f32, starts [S, n] f32 (CUDA) -> (lam [N,S], x [N,S,n], iters [N,S] i32, conv [N,S] u8)."""
        torch = _torch()
        N, S = int(entries.shape[0]), int(starts.shape[0])
        pe = _dev(entries, torch.float32, (N, self.U), "entries")
        ps = _dev(starts, torch.float32, (S, self.n), "starts")
        dev = entries.device
        if out is None:
            out = (torch.empty((N, S), dtype=torch.float32, device=dev),
                   torch.empty((N, S, self.n), dtype=torch.float32, device=dev),
                   torch.empty((N, S), dtype=torch.int32, device=dev),
                   torch.empty((N, S), dtype=torch.uint8, device=dev))
        lam, x, it, cv = out
        args = (_dev(lam, torch.float32, (N, S), "out_lambda"), _dev(x, torch.float32, (N, S, self.n), "out_x"),
                _dev(it, torch.int32, (N, S), "out_iters"), _dev(cv, torch.uint8, (N, S), "out_converged"))
        wsp, wsb = self._workspace(N, S, dev, stream) if N > 0 else (None, 0)
        opts = _Opts(int(refill_threshold), int(ctas_per_sm), None, wsp, wsb, int(schedule), 0)
        opts.chunk_tensors = int(chunk_tensors)
        alpha = self._alpha_opts(alpha, N, opts)
        if total_iters is not None:
            if total_iters.dtype != torch.int64 or not total_iters.is_cuda or total_iters.numel() != 1:
                raise TypeError("total_iters must be a 1-element int64 CUDA tensor")
            opts.d_total_iters = total_iters.data_ptr()
        _check(lib().sshopm_solve_ex(self._h, N, pe, S, ps, float(alpha), float(tol), int(maxit), *args,
                                     ctypes.byref(opts), _stream(stream)), "sshopm_solve")
        return out

    def solve_plain(self, entries, starts, alpha=0.0, tol=1e-6, maxit=100, out=None, stream=None):
        """The sshopm_solve entry point itself: library defaults, a workspace the library
        allocates and frees on the stream (cudaMallocAsync), scalar alpha only."""
        torch = _torch()
        N, S = int(entries.shape[0]), int(starts.shape[0])
        pe = _dev(entries, torch.float32, (N, self.U), "entries")
        ps = _dev(starts, torch.float32, (S, self.n), "starts")
        dev = entries.device
        if out is None:
            out = (torch.empty((N, S), dtype=torch.float32, device=dev),
                   torch.empty((N, S, self.n), dtype=torch.float32, device=dev),
                   torch.empty((N, S), dtype=torch.int32, device=dev),
                   torch.empty((N, S), dtype=torch.uint8, device=dev))
        lam, x, it, cv = out
        _check(lib().sshopm_solve(self._h, N, pe, S, ps, float(alpha), float(tol), int(maxit),
                                  _dev(lam, torch.float32, (N, S), "out_lambda"),
                                  _dev(x, torch.float32, (N, S, self.n), "out_x"),
                                  _dev(it, torch.int32, (N, S), "out_iters"),
                                  _dev(cv, torch.uint8, (N, S), "out_converged"), _stream(stream)), "sshopm_solve")
        return out

    def solve_dedup(self, entries, starts, alpha=0.0, tol=1e-6, maxit=100, lam_tol=1e-2, ang_tol=0.05, kmax=8,
                    out=None, dedup_out=None, refill_threshold=0, ctas_per_sm=0, total_iters=None, stream=None,
                    schedule=0, fused=False, records_only=False, warp_specialized=False, records=False,
                    unit_starts=0):
        """Fused solve + dedup (sshopm_solve_dedup).  Returns (raw outputs, dedup outputs) as in solve() / dedup().
        fused: cluster inside the solve kernel (schedule 1 ring, or schedule 7 staging).  records_only: the
        schedule-7 pipeline clusters in-kernel and leaves the raw outputs unwritten (they are scratch).
        warp_specialized: one warp per CTA of the solve kernel clusters the chunks the other seven complete.
        records: the records path (schedule 8, fuse_dedup = 4): lanes own units of `unit_starts` starts of one
        tensor, per-start results go to a 16-byte record scratch the dedup reads; no raw outputs (returns
        (None, dedup outputs))."""
        torch = _torch()
        N, S = int(entries.shape[0]), int(starts.shape[0])
        pe = _dev(entries, torch.float32, (N, self.U), "entries")
        ps = _dev(starts, torch.float32, (S, self.n), "starts")
        dev = entries.device
        if records:
            if dedup_out is None:
                dedup_out = (torch.empty((N,), dtype=torch.int32, device=dev),
                             torch.empty((N, kmax), dtype=torch.float32, device=dev),
                             torch.empty((N, kmax, self.n), dtype=torch.float32, device=dev),
                             torch.empty((N, kmax), dtype=torch.int32, device=dev),
                             torch.empty((N, kmax), dtype=torch.int32, device=dev))
            c, ol, ox, om, orp = dedup_out
            dargs = (_dev(c, torch.int32, (N,), "out_count"), _dev(ol, torch.float32, (N, kmax), "out_clambda"),
                     _dev(ox, torch.float32, (N, kmax, self.n), "out_cx"), _dev(om, torch.int32, (N, kmax), "out_mult"),
                     _dev(orp, torch.int32, (N, kmax), "out_rep"))
            wsp, wsb = self._workspace(N, S, dev, stream) if N > 0 else (None, 0)
            rp, rb = self._records(N, S, dev, stream) if N > 0 else (None, 0)
            opts = _Opts(int(refill_threshold), int(ctas_per_sm), None, wsp, wsb, int(schedule), 4)
            opts.d_records, opts.records_bytes, opts.unit_starts = rp, rb, int(unit_starts)
            alpha = self._alpha_opts(alpha, N, opts)
            if total_iters is not None:
                opts.d_total_iters = total_iters.data_ptr()
            _check(lib().sshopm_solve_dedup(self._h, N, pe, S, ps, float(alpha), float(tol), int(maxit), None, None,
                                            None, None, float(lam_tol), float(ang_tol), int(kmax), *dargs,
                                            ctypes.byref(opts), _stream(stream)), "sshopm_solve_dedup")
            return None, dedup_out
        if out is None:
            out = (torch.empty((N, S), dtype=torch.float32, device=dev),
                   torch.empty((N, S, self.n), dtype=torch.float32, device=dev),
                   torch.empty((N, S), dtype=torch.int32, device=dev),
                   torch.empty((N, S), dtype=torch.uint8, device=dev))
        if dedup_out is None:
            dedup_out = (torch.empty((N,), dtype=torch.int32, device=dev),
                         torch.empty((N, kmax), dtype=torch.float32, device=dev),
                         torch.empty((N, kmax, self.n), dtype=torch.float32, device=dev),
                         torch.empty((N, kmax), dtype=torch.int32, device=dev),
                         torch.empty((N, kmax), dtype=torch.int32, device=dev))
        lam, x, it, cv = out
        c, ol, ox, om, orp = dedup_out
        args = (_dev(lam, torch.float32, (N, S), "out_lambda"), _dev(x, torch.float32, (N, S, self.n), "out_x"),
                _dev(it, torch.int32, (N, S), "out_iters"), _dev(cv, torch.uint8, (N, S), "out_converged"))
        dargs = (_dev(c, torch.int32, (N,), "out_count"), _dev(ol, torch.float32, (N, kmax), "out_clambda"),
                 _dev(ox, torch.float32, (N, kmax, self.n), "out_cx"), _dev(om, torch.int32, (N, kmax), "out_mult"),
                 _dev(orp, torch.int32, (N, kmax), "out_rep"))
        wsp, wsb = self._workspace(N, S, dev, stream) if N > 0 else (None, 0)
        opts = _Opts(int(refill_threshold), int(ctas_per_sm), None, wsp, wsb, int(schedule),
                     3 if warp_specialized else (2 if records_only else (1 if fused else 0)))
        alpha = self._alpha_opts(alpha, N, opts)
        if total_iters is not None:
            opts.d_total_iters = total_iters.data_ptr()
        _check(lib().sshopm_solve_dedup(self._h, N, pe, S, ps, float(alpha), float(tol), int(maxit), *args,
                                        float(lam_tol), float(ang_tol), int(kmax), *dargs, ctypes.byref(opts),
                                        _stream(stream)), "sshopm_solve_dedup")
        return out, dedup_out

    def dedup(self, lam, x, conv, lam_tol=1e-2, ang_tol=0.05, kmax=8, out=None, stream=None):
        """-> (count [N] i32, lam [N,kmax], x [N,kmax,n], mult [N,kmax] i32, rep [N,kmax] i32)."""
        torch = _torch()
        N, S = int(lam.shape[0]), int(lam.shape[1])
        pl = _dev(lam, torch.float32, (N, S), "lambda")
        px = _dev(x, torch.float32, (N, S, self.n), "x")
        pc = _dev(conv, torch.uint8, (N, S), "converged")
        dev = lam.device
        if out is None:
            out = (torch.empty((N,), dtype=torch.int32, device=dev),
                   torch.empty((N, kmax), dtype=torch.float32, device=dev),
                   torch.empty((N, kmax, self.n), dtype=torch.float32, device=dev),
                   torch.empty((N, kmax), dtype=torch.int32, device=dev),
                   torch.empty((N, kmax), dtype=torch.int32, device=dev))
        c, ol, ox, om, orp = out
        _check(lib().sshopm_dedup(self._h, N, S, pl, px, pc, float(lam_tol), float(ang_tol), int(kmax),
                                  _dev(c, torch.int32, (N,), "out_count"),
                                  _dev(ol, torch.float32, (N, kmax), "out_lambda"),
                                  _dev(ox, torch.float32, (N, kmax, self.n), "out_x"),
                                  _dev(om, torch.int32, (N, kmax), "out_mult"),
                                  _dev(orp, torch.int32, (N, kmax), "out_rep"), _stream(stream)), "sshopm_dedup")
        return out

    def classify(self, entries, count, lam, x, ctol=1e-3, stream=None):
        """Eigenpair types [N, kmax] int8 of dedup records: +1 max, -1 min, 0 saddle, 2 degenerate, 3 empty."""
        torch = _torch()
        N, K = int(lam.shape[0]), int(lam.shape[1])
        out = torch.empty((N, K), dtype=torch.int8, device=lam.device)
        _check(lib().sshopm_classify(self._h, N, _dev(entries, torch.float32, (N, self.U), "entries"), K,
                                     _dev(count, torch.int32, (N,), "count"), _dev(lam, torch.float32, (N, K), "lambda"),
                                     _dev(x, torch.float32, (N, K, self.n), "x"), float(ctol),
                                     ctypes.c_void_p(out.data_ptr()), _stream(stream)), "sshopm_classify")
        return out

    def apply(self, entries, x, stream=None):
        """Test hook: (A x^{m-1} [N, n], A x^m [N]) with the solver's compiled evaluation."""
        torch = _torch()
        N = int(entries.shape[0])
        pe = _dev(entries, torch.float32, (N, self.U), "entries")
        px = _dev(x, torch.float32, (N, self.n), "x")
        g = torch.empty((N, self.n), dtype=torch.float32, device=entries.device)
        lam = torch.empty((N,), dtype=torch.float32, device=entries.device)
        _check(lib().sshopm_apply(self._h, N, pe, px, ctypes.c_void_p(g.data_ptr()), ctypes.c_void_p(lam.data_ptr()),
                                  _stream(stream)), "sshopm_apply")
        return g, lam

    def run_host(self, entries, starts, alpha=0.0, tol=1e-6, maxit=100, lam_tol=1e-2, ang_tol=0.05, kmax=8,
                 raw=False, chunk_tensors=0, out=None):
        """End-to-end on HOST arrays (numpy or pinned CPU torch tensors); returns a dict of host arrays.
        A caller-provided `out` without "rep" skips the representative-start field (d_out_rep = NULL)."""
        def ptr(a, dtype, shape, name):
            """Host pointer of `a` after checking dtype, shape and layout (the C ABI reads raw memory)."""
            if hasattr(a, "data_ptr"):
                torch = _torch()
                tdt = {np.float32: torch.float32, np.int32: torch.int32, np.uint8: torch.uint8}[dtype]
                if a.is_cuda:
                    raise TypeError(f"{name} must be a host (CPU) tensor")
                if a.dtype != tdt:
                    raise TypeError(f"{name} must be {tdt}, got {a.dtype}")
                if tuple(a.shape) != tuple(shape):
                    raise ValueError(f"{name} must have shape {tuple(shape)}, got {tuple(a.shape)}")
                if not a.is_contiguous():
                    raise ValueError(f"{name}: host tensors must be contiguous")
                return ctypes.c_void_p(a.data_ptr())
            if not isinstance(a, np.ndarray):
                raise TypeError(f"{name} must be a numpy array or a CPU torch tensor")
            if a.dtype != np.dtype(dtype):
                raise TypeError(f"{name} must be {np.dtype(dtype)}, got {a.dtype}")
            if tuple(a.shape) != tuple(shape):
                raise ValueError(f"{name} must have shape {tuple(shape)}, got {tuple(a.shape)}")
            if not a.flags["C_CONTIGUOUS"]:
                raise ValueError(f"{name}: host arrays must be C-contiguous")
            return ctypes.c_void_p(a.ctypes.data)

        N, S = int(entries.shape[0]), int(starts.shape[0])
        if out is None:
            out = {"count": np.empty(N, np.int32), "lambda": np.empty((N, kmax), np.float32),
                   "x": np.empty((N, kmax, self.n), np.float32), "mult": np.empty((N, kmax), np.int32),
                   "rep": np.empty((N, kmax), np.int32)}
            if raw:
                out.update({"raw_lambda": np.empty((N, S), np.float32), "raw_x": np.empty((N, S, self.n), np.float32),
                            "raw_iters": np.empty((N, S), np.int32), "raw_converged": np.empty((N, S), np.uint8)})
        n, K, f4, i4, u1 = self.n, int(kmax), np.float32, np.int32, np.uint8
        pe = ptr(entries, f4, (N, self.U), "entries")
        ps = ptr(starts, f4, (S, n), "starts")
        rawspec = {"raw_lambda": (f4, (N, S)), "raw_x": (f4, (N, S, n)), "raw_iters": (i4, (N, S)),
                   "raw_converged": (u1, (N, S))}
        rawp = [ptr(out[k], *rawspec[k], k) if raw else None for k in rawspec]
        rp = ptr(out["rep"], i4, (N, K), "rep") if out.get("rep") is not None else None
        tot = ctypes.c_ulonglong(0)
        _check(lib().sshopm_run_host(self._h, N, pe, S, ps, float(alpha), float(tol), int(maxit),
                                     float(lam_tol), float(ang_tol), K, ptr(out["count"], i4, (N,), "count"),
                                     ptr(out["lambda"], f4, (N, K), "lambda"), ptr(out["x"], f4, (N, K, n), "x"),
                                     ptr(out["mult"], i4, (N, K), "mult"), rp,
                                     *rawp, int(chunk_tensors),
                                     ctypes.byref(tot)), "sshopm_run_host")
        out["total_iters"] = tot.value
        return out
