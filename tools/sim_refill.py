"""Trace-driven simulation of the solve kernel's lane scheduling: per-lane evaluation counts
(iters + 1) come from the FP64 oracle on synthetic (4,3) tensors; a warp of 32 lanes (x slots) processes
items and is refilled by the policies below.  Reports lane utilisation (useful lane-steps / lane-steps) and,
with instruction costs per step / refill, an efficiency against the bare step.

    python tools/sim_refill.py [tensors]          # oracle run on `tensors` x 128 starts (default 1024)

Policies: item (schedule 1: refill when >= K lanes stopped, every STEPS steps), pair (two slots per lane
refilled together with two starts of one tensor), pool (two slots, per-slot refill from the lane's tensor).
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def iteration_counts(tensors):
    import synthetic as syn
    from oracle import sshopm as O
    ent = syn.gen_voxels(4, 3, 0, tensors, seed=0)
    st = syn.gen_starts(128, 3, seed=0)
    return (O.sshopm(ent, st, 4, 3, 0.0, 1e-6, 100)[2] + 1).astype(np.int64)


def item_policy(ev, K, STEPS, c_step=61, c_ref=73, c_chk=4, nwarps=8):
    items = ev.reshape(-1)
    per = len(items) // nwarps
    steps = useful = refills = trips = 0
    for w in range(nwarps):
        q, qi = items[w * per:(w + 1) * per], 0
        rem = np.zeros(32, np.int64)
        while True:
            stopped = rem == 0
            cnt = int(stopped.sum())
            if (cnt >= K or qi >= len(q)) and cnt:
                if qi < len(q):
                    idx = np.nonzero(stopped)[0][:len(q) - qi]
                    rem[idx] = q[qi:qi + len(idx)]
                    qi += len(idx)
                    refills += 1
                if qi >= len(q) and rem.sum() == 0:
                    break
            trips += 1
            for _ in range(STEPS):
                a = rem > 0
                useful += int(a.sum())
                rem[a] -= 1
                steps += 1
    cost = steps * c_step + refills * c_ref + trips * c_chk
    return useful / (32 * steps), useful / 32 * c_step / cost


def pair_policy(ev, K, STEPS, nwarps=8):
    pairs = ev.reshape(-1, 2)
    per = len(pairs) // nwarps
    steps = useful = 0
    for w in range(nwarps):
        q, qi = pairs[w * per:(w + 1) * per], 0
        rem = np.zeros((32, 2), np.int64)
        while True:
            stopped = (rem == 0).all(1)
            cnt = int(stopped.sum())
            if (cnt >= K or qi >= len(q)) and cnt:
                if qi < len(q):
                    idx = np.nonzero(stopped)[0][:len(q) - qi]
                    rem[idx] = q[qi:qi + len(idx)]
                    qi += len(idx)
                if qi >= len(q) and rem.sum() == 0:
                    break
            for _ in range(STEPS):
                a = rem > 0
                useful += int(a.sum())
                rem[a] -= 1
                steps += 1
    return useful / (64 * steps)


def pool_policy(ev, STEPS, nwarps=8):
    T, S = ev.shape
    per = T // nwarps
    steps = useful = 0
    for w in range(nwarps):
        tq, ti, p = list(range(w * per, (w + 1) * per)), 0, 0
        rem = np.zeros((32, 2), np.int64)
        bind = np.full(32, -1)
        while True:
            for l in range(32):
                if ti >= len(tq):
                    break
                if (rem[l] == 0).all() and bind[l] != ti:
                    bind[l] = ti
                if bind[l] == ti:
                    for sl in range(2):
                        if rem[l, sl] == 0 and ti < len(tq):
                            rem[l, sl] = ev[tq[ti], p]
                            p += 1
                            if p == S:
                                ti, p = ti + 1, 0
            if ti >= len(tq) and (rem == 0).all():
                break
            for _ in range(STEPS):
                a = rem > 0
                useful += int(a.sum())
                rem[a] -= 1
                steps += 1
    return useful / (64 * steps)


def affinity_policy(ev, K, STEPS, nwarps=8):
    """Two slots per lane, the lane owns one tensor at a time: when >= K of the warp's 64 slots are stopped,
    every stopped slot takes its lane's tensor's next start; a lane whose tensor has no start left and whose
    two slots are both stopped claims the next tensor (coefficient reload).  Returns (utilisation, refill
    events per useful slot-step, tensor switches per useful slot-step)."""
    T, S = ev.shape
    per = T // nwarps
    steps = useful = refills = switches = 0
    for w in range(nwarps):
        nxt_t = w * per
        end_t = (w + 1) * per
        ten = np.full(32, -1)
        pos = np.full(32, S)
        rem = np.zeros((32, 2), np.int64)
        while True:
            stopped = rem == 0
            cnt = int(stopped.sum())
            live = (pos < S).any() or nxt_t < end_t
            if (cnt >= K or not live) and cnt:
                refills += 1
                for l in range(32):
                    if pos[l] >= S and stopped[l].all() and nxt_t < end_t:
                        ten[l], pos[l] = nxt_t, 0
                        nxt_t += 1
                        switches += 1
                    for sl in range(2):
                        if rem[l, sl] == 0 and pos[l] < S:
                            rem[l, sl] = ev[ten[l], pos[l]]
                            pos[l] += 1
                if not live and rem.sum() == 0:
                    break
            for _ in range(STEPS):
                a = rem > 0
                useful += int(a.sum())
                rem[a] -= 1
                steps += 1
    return useful / (64 * steps), refills / useful, switches / useful


def main_affinity():
    ev = iteration_counts(int(sys.argv[2]) if len(sys.argv) > 2 else 1024)
    for K, ST in [(8, 2), (12, 2), (16, 2), (12, 3), (16, 3), (20, 3), (24, 4), (16, 4)]:
        u, r, s = affinity_policy(ev, K, ST)
        print(f"affinity K={K} STEPS={ST}: slot utilisation {u:.3f}, refill events per useful slot-step {r:.4f}, "
              f"tensor switches per useful slot-step {s:.5f}")
    for K, ST in [(10, 4), (8, 3)]:
        u, e = item_policy(ev, K, ST)
        print(f"item  K={K} STEPS={ST}: lane utilisation {u:.3f}")


if __name__ == "__main__" and sys.argv[1:2] == ["affinity"]:
    main_affinity()
elif __name__ == "__main__":
    ev = iteration_counts(int(sys.argv[1]) if len(sys.argv) > 1 else 1024)
    print(f"mean evaluations per item {ev.mean():.2f}, p99 {np.percentile(ev, 99):.0f}")
    for K, ST in [(8, 3), (6, 3), (4, 3), (4, 1)]:
        u, e = item_policy(ev, K, ST)
        print(f"item  K={K} STEPS={ST}: lane utilisation {u:.3f}, efficiency vs bare step {e:.3f}")
    for K, ST in [(2, 1), (4, 2), (8, 3)]:
        print(f"pair  K={K} STEPS={ST}: lane utilisation {pair_policy(ev, K, ST):.3f}")
    for ST in (1, 2):
        print(f"pool  STEPS={ST}: lane utilisation {pool_policy(ev, ST):.3f}")
