"""Culling-granularity simulation (CPU): evaluated / within for per-atom box tests at several item-group sizes."""
import sys
import numpy as np
sys.path.insert(0, "/root/repo")
from paper_conf_ppopp_imbernoncg16_b200 import synth


def quat_rot(q):
    w, x, y, z = q.T
    return np.stack([
        np.stack([1 - 2 * (y * y + z * z), 2 * (x * y - w * z), 2 * (x * z + w * y)], -1),
        np.stack([2 * (x * y + w * z), 1 - 2 * (x * x + z * z), 2 * (y * z - w * x)], -1),
        np.stack([2 * (x * z - w * y), 2 * (y * z + w * x), 1 - 2 * (x * x + y * y)], -1)], -2)


def hilbert_key(p, bits=10):
    # Morton key of a fine grid (close enough to Hilbert for box statistics)
    lo = p.min(0)
    g = ((p - lo) / 0.25).astype(np.int64)
    k = np.zeros(len(p), np.int64)
    for b in range(bits):
        for d in range(3):
            k |= ((g[:, d] >> b) & 1) << (3 * b + d)
    return k


def box_dist2(lo, hi, a):
    d = np.maximum(0, np.maximum(lo[None] - a, a - hi[None]))
    return (d * d).sum(1)


name = sys.argv[1] if len(sys.argv) > 1 else "medium"
P = int(sys.argv[2]) if len(sys.argv) > 2 else 256
prob = synth.make_problem(name)
rc = 12.0
rng = np.random.default_rng(0)
rec = prob.rec.xyz.astype(np.float64)
lig = prob.lig.xyz.astype(np.float64)
res = {}
for s in range(0, prob.cfg.n_spots, max(1, prob.cfg.n_spots // 6)):
    c = prob.spots[s].astype(np.float64)
    q = rng.normal(size=(P, 4)); q /= np.linalg.norm(q, axis=1, keepdims=True)
    t = rng.uniform(-3, 3, (P, 3))
    items = (c + t)[:, None, :] + np.einsum("pij,aj->pai", quat_rot(q), lig)
    items = items.reshape(-1, 3)
    items = items[np.argsort(hilbert_key(items), kind="stable")]
    lst = rec[np.linalg.norm(rec - c, axis=1) < rc + 3 + 10]
    for gi in [64, 32, 16, 8]:
        ev = wi = 0
        for b in range(0, len(items) - 63, 64):
            blk = items[b:b + 64]
            mx = 0
            for sb in range(0, 64, gi):
                sub = blk[sb:sb + gi]
                n = (box_dist2(sub.min(0), sub.max(0), lst) < rc * rc).sum()
                mx = max(mx, n)
            ev += 64 * mx
            if gi == 64:
                d2 = ((blk[:, None, :] - lst[None]) ** 2).sum(-1)
                wi += (d2 < rc * rc).sum()
        res.setdefault(gi, [0, 0])
        res[gi][0] += ev
        if gi == 64:
            w_tot = res.setdefault("w", [0])
            w_tot[0] += wi
for gi in [64, 32, 16, 8]:
    print(f"{name} P{P}: group {gi} items -> evaluated / within {res[gi][0] / res['w'][0]:.3f}")
