"""Per-voxel eigenpair dedup / clustering oracle — TEST INFRASTRUCTURE ONLY.

The paper runs SS-HOPM from many starts to find "one or more eigenpairs for
each tensor" whose local maxima are the fibre directions
 but gives no rule for merging the per-start results.
DESIGN.md reading R16 fixes one, written out here literally:

* only converged starts take part, visited in start order;
* a start joins the FIRST existing cluster (creation order) whose
  representative r satisfies |lam_s - lam_r| <= lam_tol * max(1, |lam_r|) and
  angle(x_s, x_r) <= ang_tol, the angle being sign-free for even m (x and -x
  are the same eigenvector, reading R15); for odd m, (lam, x) ~ (-lam, -x) is
  accepted as the same eigenpair as well;
* otherwise it founds a new cluster and is its representative;
* clusters are reported by representative lam descending, ties by
  representative start index ascending; ``count`` is the total number of
  clusters (it may exceed kmax — overflow), the first kmax are stored;
  empty slots hold lam = 0, x = 0, mult = 0, rep = -1.

The angle uses Kahan's stable form 2*atan2(||a-b||, ||a+b||) on unit vectors.
The count is bounded by ((m-1)^n - 1)/(m-2) distinct eigenpairs only
when the clusters are true distinct eigenpairs; tests use that as a pin.
"""
import numpy as np


def angle(a, b):
    """Angle between vectors a and b (radians), FP64, stable for small angles."""
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    a = a / np.linalg.norm(a)
    b = b / np.linalg.norm(b)
    return 2.0 * np.arctan2(np.linalg.norm(a - b), np.linalg.norm(a + b))


def same_pair(lam_s, x_s, lam_r, x_r, m, lam_tol, ang_tol):
    """Reading R16 membership test against representative (lam_r, x_r)."""
    def close(ls, xs):
        return abs(ls - lam_r) <= lam_tol * max(1.0, abs(lam_r)) and angle(xs, x_r) <= ang_tol

    if m % 2 == 0:
        return close(lam_s, x_s) or close(lam_s, -np.asarray(x_s))
    return close(lam_s, x_s) or close(-lam_s, -np.asarray(x_s))


def dedup_voxel(lam, x, conv, m, lam_tol, ang_tol):
    """Greedy clustering of one voxel's S results. Returns list of (rep, mult), unsorted."""
    reps, mult = [], []
    for s in range(len(lam)):
        if not conv[s]:
            continue
        for c, r in enumerate(reps):
            if same_pair(lam[s], x[s], lam[r], x[r], m, lam_tol, ang_tol):
                mult[c] += 1
                break
        else:
            reps.append(s)
            mult.append(1)
    return reps, mult


def dedup(lam, x, conv, m, lam_tol, ang_tol, kmax):
    """Batched reading-R16 dedup.

    lam [V,S], x [V,S,n], conv [V,S].  Returns count [V] int32, lam_out [V,kmax],
    x_out [V,kmax,n], mult [V,kmax] int32, rep [V,kmax] int32.
    """
    lam = np.asarray(lam, np.float64)
    x = np.asarray(x, np.float64)
    conv = np.asarray(conv).astype(bool)
    V, S = lam.shape
    n = x.shape[2]
    count = np.zeros(V, np.int32)
    lo = np.zeros((V, kmax))
    xo = np.zeros((V, kmax, n))
    mo = np.zeros((V, kmax), np.int32)
    ro = np.full((V, kmax), -1, np.int32)
    for v in range(V):
        reps, mult = dedup_voxel(lam[v], x[v], conv[v], m, lam_tol, ang_tol)
        order = sorted(range(len(reps)), key=lambda c: (-lam[v, reps[c]], reps[c]))
        count[v] = len(reps)
        for slot, c in enumerate(order[:kmax]):
            r = reps[c]
            lo[v, slot] = lam[v, r]
            xo[v, slot] = x[v, r]
            mo[v, slot] = mult[c]
            ro[v, slot] = r
    return count, lo, xo, mo, ro
