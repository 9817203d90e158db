#!/usr/bin/env python
"""Offline study: list atoms streamed per item for 128-item chunks sorted by Morton vs Hilbert (16^3 cells), medium
config, exact box culling (no cell rows).  Reproduces the numbers in profiles/r01_notes.md."""
import sys, numpy as np
sys.path.insert(0, __import__('os').path.dirname(__import__('os').path.dirname(__import__('os').path.abspath(__file__))))
from paper_conf_ppopp_imbernoncg16_b200 import synth
from scipy.spatial.transform import Rotation as Rot
prob = synth.make_problem('medium')
lig = prob.lig.xyz - prob.lig.xyz.mean(0)
rec = prob.rec.xyz
rng = np.random.default_rng(0)

def spread(v):
    out = np.zeros_like(v)
    for b in range(4): out |= ((v >> b) & 1) << (3 * b)
    return out

def hilbert3(x, y, z, bits=4):
    # Skilling's AxesToTranspose then interleave
    X = [x.copy(), y.copy(), z.copy()]
    n = 3; M = 1 << (bits - 1)
    Q = M
    while Q > 1:
        P = Q - 1
        for i in range(n):
            m = (X[i] & Q) != 0
            X[0] = np.where(m, X[0] ^ P, X[0])
            t = (X[0] ^ X[i]) & P
            X[0] = np.where(m, X[0], X[0] ^ t)
            X[i] = np.where(m, X[i], X[i] ^ t)
        Q >>= 1
    for i in range(1, n): X[i] ^= X[i - 1]
    t = np.zeros_like(x); Q = M
    while Q > 1:
        t = np.where((X[n - 1] & Q) != 0, t ^ (Q - 1), t); Q >>= 1
    for i in range(n): X[i] ^= t
    key = np.zeros_like(x)
    for b in range(bits - 1, -1, -1):
        for i in range(n):
            key = (key << 1) | ((X[i] >> b) & 1)
    return key

rc = 12.0
tot = {'morton': [], 'hilbert': []}
for s in range(0, 500, 50):
    c = prob.spots[s]
    P = 256
    # a converged-ish population: poses concentrated (t within 1.5 A, random rotations) and a random one
    for spreadT in (3.0, 1.0):
        t = rng.uniform(-spreadT, spreadT, size=(P, 3))
        R = Rot.random(P, random_state=rng.integers(1 << 30)).as_matrix()
        items = (np.einsum('pij,aj->pai', R, lig) + t[:, None, :]).reshape(-1, 3)
        W = 3 + np.linalg.norm(lig, axis=1).max() + 0.01
        m = np.clip(((items + W) / (2 * W) * 16).astype(np.int64), 0, 15)
        keys = {'morton': spread(m[:, 0]) | (spread(m[:, 1]) << 1) | (spread(m[:, 2]) << 2),
                'hilbert': hilbert3(m[:, 0], m[:, 1], m[:, 2])}
        lst = rec - c
        lst = lst[np.linalg.norm(lst, axis=1) <= 3 * np.sqrt(3) + np.linalg.norm(lig, axis=1).max() + rc + 0.01]
        for name, k in keys.items():
            o = np.argsort(k, kind='stable')
            it = items[o]
            ev = 0
            for a in range(0, len(it), 128):
                ch = it[a:a + 128]
                lo, hi = ch.min(0), ch.max(0)
                d = np.maximum(0, np.maximum(lo - lst, lst - hi))
                ev += len(ch) * np.sum((d ** 2).sum(1) < (rc + 0.01) ** 2)
            tot[name].append((spreadT, ev / (len(items) * len(lst))))
for name in tot:
    a = np.array(tot[name])
    for sp in (3.0, 1.0):
        print(name, 'spread', sp, 'streamed fraction %.4f' % a[a[:, 0] == sp, 1].mean())
