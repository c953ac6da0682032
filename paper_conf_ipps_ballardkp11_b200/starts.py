"""Starting vectors for SS-HOPM.

"We choose random vectors by independently selecting each vector entry
uniformly from [-1, 1] and then normalizing.  Alternatively, one could use a
deterministic approach and pick starting vectors evenly spaced about the
sphere."  Both are provided as host arrays of shape [S, n] (float32); the
solver normalises them on the device (reading R7), so these need not be unit.

* ``uniform_cube(S, n, seed)``   — the paper's random starts.
* ``evenly_spaced(S, n, half)``  — deterministic: the spherical Fibonacci
  lattice for n = 3 (n = 2: equal angles), for other n a Halton sequence
  mapped to the sphere through the Gaussian (Box-Muller) construction.  With
  ``half=True`` points are spread over a hemisphere, which covers the sphere
  for even m where x and -x are the same eigenvector (reading R15).
"""
import math

import numpy as np


def uniform_cube(S, n, seed=0):
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x57A27, S, n])))
    return rng.uniform(-1.0, 1.0, size=(S, n)).astype(np.float32)


def _primes(k):
    out, c = [], 2
    while len(out) < k:
        if all(c % p for p in out):
            out.append(c)
        c += 1
    return out


def _halton(S, dims):
    pts = np.zeros((S, dims))
    for d, b in enumerate(_primes(dims)):
        for i in range(S):
            f, r, j = 1.0, 0.0, i + 1
            while j > 0:
                f /= b
                r += f * (j % b)
                j //= b
            pts[i, d] = r
    return pts


def evenly_spaced(S, n, half=False):
    """float32 [S, n] deterministic, approximately evenly spaced unit vectors."""
    if S < 1 or n < 1:
        raise ValueError("S and n must be positive")
    if n == 1:
        return np.ones((S, 1), np.float32)
    if n == 2:
        span = math.pi if half else 2 * math.pi
        t = (np.arange(S) + 0.5) / S * span
        return np.stack([np.cos(t), np.sin(t)], 1).astype(np.float32)
    if n == 3:
        i = np.arange(S) + 0.5
        z = 1 - (i / S) * (1.0 if half else 2.0)          # half: z in (0, 1]
        r = np.sqrt(np.maximum(0.0, 1 - z * z))
        phi = math.pi * (1 + 5 ** 0.5) * i
        return np.stack([r * np.cos(phi), r * np.sin(phi), z], 1).astype(np.float32)
    # n >= 4: Halton -> Gaussian (Box-Muller) -> sphere
    dims = n + (n % 2)
    h = _halton(S, dims)
    u1 = np.clip(h[:, 0::2], 1e-12, 1.0)
    u2 = h[:, 1::2]
    g = np.sqrt(-2 * np.log(u1))
    z = np.concatenate([g * np.cos(2 * math.pi * u2), g * np.sin(2 * math.pi * u2)], 1)[:, :n]
    z /= np.linalg.norm(z, axis=1, keepdims=True)
    if half:
        z *= np.where(z[:, -1:] < 0, -1.0, 1.0)
    return z.astype(np.float32)
