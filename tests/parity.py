"""GPU-vs-oracle parity contract (readings P1-P5).

GPU: FP32 compressed evaluation.  Oracle: FP64 full tensor, same FP32 inputs.

Witnesses.  Some lanes follow non-contractive trajectories (alpha below the
convexity bound, e.g. alpha = 0 near a negative eigenvalue, "no proof of
convergence for alpha = 0"): there FP32 and FP64 rounding alone decide the
outcome.  Witness runs are the oracle's own algorithm (a) in FP32 arithmetic
(the paper's precision) and (b) in FP64 from 8 perturbations of x_0 by
2^-24 relative.  A lane is *precision-sensitive* when a witness moves the
oracle's result, or when its trajectory is ill-conditioned: some witness
lambda_k departs from the FP64 lambda_k by more than COND_LAM = 1e-5 (relative,
~100x FP32 rounding), or some witness x_k from x_k by more than COND_ANG = 1e-4
rad (~1000x FP32 rounding), at an iteration up to where the two sides stopped.
Differences on such lanes are *explained*; explained lanes are counted and must
stay rare.

P1 Converged flags identical.  A mismatch is explained iff the lane is at the
   stopping-rule boundary — the oracle's r_k = |lam_k - lam_{k-1}| /
   (tol max(1,|lam_k|)) is in [0.5, 2] at the iteration where the converged
   side stopped or at k = maxit — or a witness flips the oracle's flag.
P2 |lam_gpu - lam_ref| <= 1e-4 max(1, |lam_ref|) on lanes converged in both;
   a violation is explained iff the GPU pair has FP64 residual <= 0.05 and a
   witness moves the oracle's lambda by > 1e-4 relative, or the lane is at the
   stopping boundary (oracle r_k in [0.5, 2] at the GPU's stop k) and the
   oracle's lambda_k at that same k agrees within 1e-4 (slowly converging lanes
   where FP32 rounding moves the stop by many updates).
P3 Eigenvector angle <= 1e-3 rad between x_gpu and the oracle iterate at the
   GPU's own iteration count (trajectory alignment), sign-free for even m, on
   lanes converged in both and not explained under P2; a violation is
   explained iff a witness moves the oracle iterate at that k by > 1e-3 rad.
P4 Fixed-K (tol < 0): |lam_gpu - lam_ref| <= max(1e-5 max(1,|lam|), 1e3 s), s =
   max oracle lambda_K change over the witnesses.
"""
import json
import os

import numpy as np

from oracle import sshopm as O

LAM_TOL = 1e-4
ANG_TOL = 1e-3
FIXED_TOL = 1e-5
N_PERTURB = 8


def angle(a, b, even):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    a = a / np.linalg.norm(a, axis=-1, keepdims=True)
    b = b / np.linalg.norm(b, axis=-1, keepdims=True)
    t = 2 * np.arctan2(np.linalg.norm(a - b, axis=-1), np.linalg.norm(a + b, axis=-1))
    if even:
        t = np.minimum(t, np.pi - t)
    return t


def _lane_alpha(alpha, vox):
    """Scalar shift, or the per-voxel shift array indexed for these lanes."""
    return alpha if np.ndim(alpha) == 0 else np.asarray(alpha, np.float64)[vox]


def _lanes(full, vox, x0, alpha, tol, maxit, lane_maxit=None, dtype=np.float64):
    return O.sshopm_lanes(lambda idx: full[vox[idx]], x0, _lane_alpha(alpha, vox), tol, maxit, lane_maxit, dtype=dtype)


def _perturb(x0, seed, k):
    rng = np.random.default_rng(seed + 1000 * k)
    return O.normalise_starts(x0 * (1 + 2.0 ** -24 * rng.uniform(-1, 1, size=x0.shape)))


def witnesses(full, vox, x0, alpha, tol, maxit, lane_maxit=None):
    """Oracle re-runs of the given lanes: FP32 arithmetic + N_PERTURB start perturbations."""
    runs = [_lanes(full, vox, x0, alpha, tol, maxit, lane_maxit, dtype=np.float32)]
    for k in range(N_PERTURB):
        runs.append(_lanes(full, vox, _perturb(x0, 7, k), alpha, tol, maxit, lane_maxit))
    return runs


def _history(full, vox, x0, alpha, K, dtype=np.float64):
    """(lambda_k [K+1, L], x_k [K+1, L, n]) for k = 0..K of fixed-K runs (tol < 0)."""
    L, n = x0.shape
    h = np.full((K + 1, L), np.nan)
    hx = np.full((K + 1, L, n), np.nan)
    h[0] = O.axm(full[vox], x0.astype(dtype), dtype)
    hx[0] = x0
    tr = []
    O.sshopm_lanes(lambda idx: full[vox[idx]], x0, _lane_alpha(alpha, vox), -1.0, K, trace=tr, dtype=dtype)
    for kk, ids, ln, xn in tr:
        h[kk, ids] = ln
        hx[kk, ids] = xn
    return h, hx


def trajectory_deviation(full, vox, x0, alpha, K, even=True):
    """Witness deviation along the trajectory, k = 0..K:
    Dl[k, l] = max_w |lam_w(k) - lam_ref(k)| / max(1, |lam_ref(k)|),
    Dx[k, l] = max_w angle(x_w(k), x_ref(k)).
    Well-conditioned lanes stay at FP32 rounding (~1e-7); lanes whose
    trajectory amplifies rounding (non-contractive, chaotic, near a saddle or a
    basin boundary) exceed COND_LAM / COND_ANG."""
    ref, refx = _history(full, vox, x0, alpha, K)
    scale = np.maximum(1.0, np.abs(ref))
    Dl = np.zeros_like(ref)
    Dx = np.zeros_like(ref)
    runs = [(x0, np.float32)] + [(_perturb(x0, 7, k), np.float64) for k in range(N_PERTURB)]
    for xs, dt in runs:
        w, wx = _history(full, vox, xs, alpha, K, dtype=dt)
        Dl = np.maximum(Dl, np.nan_to_num(np.abs(w - ref) / scale))
        with np.errstate(invalid="ignore", divide="ignore"):
            Dx = np.maximum(Dx, np.nan_to_num(angle(wx, refx, even)))
    return Dl, Dx


COND_LAM = 1e-5   # ~100x FP32 rounding of lambda
COND_ANG = 1e-4   # ~1000x FP32 rounding of x


def ill_conditioned(full, vox, x0, alpha, kmax_lane, even=True):
    """True where the lane's trajectory amplifies rounding beyond COND_LAM / COND_ANG at some k <= kmax_lane."""
    if len(vox) == 0:
        return np.zeros(0, bool)
    K = int(max(1, kmax_lane.max()))
    Dl, Dx = trajectory_deviation(full, vox, x0, alpha, K, even)
    inside = np.arange(K + 1)[:, None] <= kmax_lane[None, :]
    return (np.max(np.where(inside, Dl, 0.0), axis=0) > COND_LAM) | (np.max(np.where(inside, Dx, 0.0), axis=0) > COND_ANG)


def solve_parity(ent, starts, m, n, alpha, tol, maxit, gpu, check_angle=True):
    """ent [V,U] f32, starts [S,n] f32, gpu = (lam, x, iters, conv) numpy [V,S,...]. Returns a report dict."""
    lam_g, x_g, it_g, cv_g = gpu
    cv_g = cv_g.astype(bool)
    V, S = lam_g.shape
    lam_r, x_r, it_r, cv_r = O.sshopm(ent, starts, m, n, alpha, tol, maxit)
    full = O.expand_full(ent, m, n)
    even = m % 2 == 0
    x0 = O.normalise_starts(starts)
    rep = {"lanes": V * S, "gpu_converged": float(cv_g.mean()), "ref_converged": float(cv_r.mean()),
           "gpu_mean_iters": float(it_g.mean()), "ref_mean_iters": float(it_r.mean()), "details": []}
    sensitive = np.zeros((V, S), bool)

    # P1 flags
    mism = np.argwhere(cv_g != cv_r)
    unexpl_flags = 0
    if len(mism):
        vox, st = mism[:, 0], mism[:, 1]
        kc = np.where(cv_g[vox, st], it_g[vox, st], it_r[vox, st]).astype(np.int64)

        def ratio_at(kk):
            kk = np.maximum(kk, 1)
            la, _, _, _ = _lanes(full, vox, x0[st], alpha, -1.0, int(kk.max()), kk)
            lb, _, _, _ = _lanes(full, vox, x0[st], alpha, -1.0, int(kk.max()), kk - 1)
            return np.abs(la - lb) / (tol * np.maximum(1.0, np.abs(la)))

        r_stop = ratio_at(kc)
        r_max = ratio_at(np.full(len(vox), maxit, np.int64))
        boundary = ((r_stop >= 0.5) & (r_stop <= 2.0)) | ((r_max >= 0.5) & (r_max <= 2.0))
        flip = np.zeros(len(vox), bool)
        for wl, wx, wi, wc in witnesses(full, vox, x0[st], alpha, tol, maxit):
            flip |= wc != cv_r[vox, st]
        flip |= ill_conditioned(full, vox, x0[st], alpha, np.maximum(it_g[vox, st], it_r[vox, st]).astype(np.int64), even)
        sensitive[vox[flip], st[flip]] = True
        ok = boundary | flip
        unexpl_flags = int(np.sum(~ok))
        rep["flag_boundary"] = int(boundary.sum())
        rep["flag_sensitive"] = int((flip & ~boundary).sum())
        for i in np.nonzero(~ok)[0][:10]:
            rep["details"].append(dict(rule="P1", voxel=int(vox[i]), start=int(st[i]), gpu_conv=bool(cv_g[vox[i], st[i]]),
                                       k_gpu=int(it_g[vox[i], st[i]]), k_ref=int(it_r[vox[i], st[i]]),
                                       r_stop=float(r_stop[i]), r_maxit=float(r_max[i]),
                                       lam_gpu=float(lam_g[vox[i], st[i]]), lam_ref=float(lam_r[vox[i], st[i]])))
    rep["flag_mismatch"] = int(len(mism))
    rep["flag_unexplained"] = unexpl_flags

    # P2 lambda at own stops
    both = cv_g & cv_r
    scale = np.maximum(1.0, np.abs(lam_r))
    dl = np.abs(lam_g.astype(np.float64) - lam_r) / scale
    viol = np.argwhere(both & (dl > LAM_TOL))
    explained = np.zeros((V, S), bool)
    unexpl_lam = 0
    if len(viol):
        vox, st = viol[:, 0], viol[:, 1]
        res = O.residual(full[vox], lam_g[vox, st].astype(np.float64), x_g[vox, st].astype(np.float64))
        sens = np.zeros(len(viol))
        for wl, wx, wi, wc in witnesses(full, vox, x0[st], alpha, tol, maxit):
            sens = np.maximum(sens, np.abs(wl.astype(np.float64) - lam_r[vox, st]) / scale[vox, st])
        cond = ill_conditioned(full, vox, x0[st], alpha, np.maximum(it_g[vox, st], it_r[vox, st]).astype(np.int64), even)
        # stopping-boundary lanes: the sides stopped at different updates of a slowly converging
        # trajectory; the oracle's ratio at the GPU's stop is in [0.5, 2] and the oracle's own
        # lambda at that update agrees (trajectory alignment, as in P3)
        kg = np.maximum(it_g[vox, st].astype(np.int64), 1)
        la, _, _, _ = _lanes(full, vox, x0[st], alpha, -1.0, int(kg.max()), kg)
        lb, _, _, _ = _lanes(full, vox, x0[st], alpha, -1.0, int(kg.max()), kg - 1)
        r_g = np.abs(la - lb) / (tol * np.maximum(1.0, np.abs(la)))
        aligned = np.abs(lam_g[vox, st] - la) / np.maximum(1.0, np.abs(la)) <= LAM_TOL
        boundary = (r_g >= 0.5) & (r_g <= 2.0) & aligned
        rep["lam_boundary"] = int(boundary.sum())
        ok = ((res <= 0.05) & ((sens > LAM_TOL) | cond)) | boundary
        explained[vox[ok], st[ok]] = True
        sensitive[vox[ok], st[ok]] = True
        unexpl_lam = int(np.sum(~ok))
        for i in np.nonzero(~ok)[0][:10]:
            rep["details"].append(dict(rule="P2", voxel=int(vox[i]), start=int(st[i]), res=float(res[i]),
                                       sens=float(sens[i]), lam_gpu=float(lam_g[vox[i], st[i]]),
                                       lam_ref=float(lam_r[vox[i], st[i]])))
    rep["lam_max_rel"] = float(dl[both & ~explained].max()) if (both & ~explained).any() else 0.0
    rep["lam_violations"] = int(len(viol))
    rep["lam_unexplained"] = unexpl_lam

    # P3 angle vs the oracle iterate at the GPU's iteration count
    if check_angle:
        sel = both & ~explained
        _, xk, _, _ = O.sshopm(ent, starts, m, n, alpha, -1.0, int(it_g.max()), lane_maxit=it_g)
        ang = np.zeros((V, S))
        if sel.any():
            ang[sel] = angle(x_g[sel], xk[sel], even)
        bad = np.argwhere(ang > ANG_TOL)
        unexpl_ang = 0
        if len(bad):
            vox, st = bad[:, 0], bad[:, 1]
            kk = it_g[vox, st].astype(np.int64)
            wmax = np.zeros(len(bad))
            for wl, wx, wi, wc in witnesses(full, vox, x0[st], alpha, -1.0, int(kk.max()), kk):
                wmax = np.maximum(wmax, angle(wx, xk[vox, st], even))
            ok = (wmax > ANG_TOL) | ill_conditioned(full, vox, x0[st], alpha, kk, even)
            sensitive[vox[ok], st[ok]] = True
            unexpl_ang = int(np.sum(~ok))
            ang_ok = ang.copy()
            ang_ok[vox[ok], st[ok]] = 0.0
            rep["angle_max_unexplained"] = float(ang_ok.max())
        rep["angle_max"] = float(ang[sel].max()) if sel.any() else 0.0
        rep["angle_max_aligned"] = float(np.where(sensitive, 0.0, ang).max())
        rep["angle_violations"] = int(len(bad))
        rep["angle_unexplained"] = unexpl_ang
    rep["sensitive_lanes"] = int(sensitive.sum())
    rep["sensitive_frac"] = float(sensitive.mean())
    return rep


def fixed_k_parity(ent, starts, m, n, alpha, K, lam_g):
    """tol < 0 runs: returns dict with max rel error and unexplained count (P4)."""
    lam_r, _, _, _ = O.sshopm(ent, starts, m, n, alpha, -1.0, K)
    scale = np.maximum(1.0, np.abs(lam_r))
    d = np.abs(lam_g.astype(np.float64) - lam_r)
    bad = np.argwhere(d > FIXED_TOL * scale)
    unexpl = 0
    if len(bad):
        vox, st = bad[:, 0], bad[:, 1]
        full = O.expand_full(ent, m, n)
        x0 = O.normalise_starts(starts)
        s = np.zeros(len(bad))
        for wl, wx, wi, wc in witnesses(full, vox, x0[st], alpha, -1.0, K):
            s = np.maximum(s, np.abs(wl.astype(np.float64) - lam_r[vox, st]))
        unexpl = int(np.sum(d[vox, st] > np.maximum(FIXED_TOL * scale[vox, st], 1e3 * s)))
    return {"max_rel": float((d / scale).max()), "outliers": int(len(bad)), "unexplained": unexpl}


def record(name, rep):
    """Save a parity report as JSON under <repo>/gpurun_out/parity/ (best effort; never fails a test)."""
    try:
        root = os.environ.get("GRAFT_REPO_ROOT") or os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        d = os.path.join(root, "gpurun_out", "parity")
        os.makedirs(d, exist_ok=True)
        safe = "".join(c if c.isalnum() or c in "-_.[]," else "_" for c in name)
        with open(os.path.join(d, safe + ".json"), "w") as f:
            json.dump(rep, f, default=lambda o: o.item() if hasattr(o, "item") else str(o))
    except OSError:
        pass
