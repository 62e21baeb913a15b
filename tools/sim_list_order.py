"""Distinct neighbour records per warp step (32 Morton-consecutive targets, one
thread per target) under several per-lane list orders: ascending (the
product), warp frequency (count of lanes holding j, descending), two classes
(held by >= 16 lanes first), partner-first (j also in lane l^1 first).  Jittered
lattice turbulence 40^3, 64 random warps.  Output in profiles/r02_sim_list_order.txt."""
import numpy as np, sys
sys.path.insert(0, __import__('os').path.dirname(__import__('os').path.dirname(__import__('os').path.abspath(__file__))))
from paper_conf_sc_simsekpc24_b200 import ics
from scipy.spatial import cKDTree
w = ics.turbulence(40)
s = w.state
x, y, z, h = (np.asarray(s[k]) for k in ('x', 'y', 'z', 'h'))
n = len(x)
# Morton sort
def spread(v):
    v = v.astype(np.uint64) & np.uint64(0x1fffff)
    for sh, m in ((32, 0x1f00000000ffff), (16, 0x1f0000ff0000ff), (8, 0x100f00f00f00f00f), (4, 0x10c30c30c30c30c3), (2, 0x1249249249249249)):
        v = (v | (v << np.uint64(sh))) & np.uint64(m)
    return v
q = lambda a: np.clip((a * (1 << 21)).astype(np.int64), 0, (1 << 21) - 1)
key = (spread(q(x % 1.0)) << np.uint64(2)) | (spread(q(y % 1.0)) << np.uint64(1)) | spread(q(z % 1.0))
o = np.argsort(key, kind='stable')
x, y, z, h = x[o], y[o], z[o], h[o]
P = np.stack([x, y, z], 1) % 1.0
T = cKDTree(P, boxsize=1.0)
rng = np.random.default_rng(0)
warps = rng.choice(n // 32, 64, replace=False)
def lists_for(w0):
    L = []
    for t in range(w0 * 32, w0 * 32 + 32):
        nb = np.array(sorted(j for j in T.query_ball_point(P[t], 2 * h[t]) if j != t))
        L.append(nb)
    return L
def distinct_per_step(L, sector=1):
    K = max(len(l) for l in L)
    tot = 0; pairs = sum(len(l) for l in L)
    for k in range(K):
        tot += len({l[k] // sector for l in L if k < len(l)})
    return tot, pairs, K
res = {}
for name in ('asc', 'countdesc', 'count2', 'partner'):
    T_, P_, S_ = 0, 0, 0
    for w0 in warps:
        L = lists_for(w0)
        if name != 'asc':
            from collections import Counter
            c = Counter(j for l in L for j in l)
            if name == 'countdesc':
                L = [np.array(sorted(l, key=lambda j: (-c[j], j))) for l in L]
            elif name == 'count2':
                L = [np.array(sorted(l, key=lambda j: (c[j] < 16, j))) for l in L]
            elif name == 'partner':
                L2 = []
                for t, l in enumerate(L):
                    p = set(L[t ^ 1])
                    L2.append(np.array(sorted(l, key=lambda j: (j not in p, j))))
                L = L2
        a, b, k = distinct_per_step(L)
        T_ += a; P_ += b; S_ += k
    res[name] = (T_ / S_, T_ / P_)
    print(name, 'distinct per step %.2f, per pair %.3f, steps/warp %.1f' % (T_ / S_, T_ / P_, S_ / len(warps)))


def hier_order(L):
    """Hierarchical: j held by every lane of the lane's aligned group of 32, then
    of 16, 8, 4, 2, then the rest; ascending j within a level.  Within an aligned
    group every lane's list starts with the same segments in the same order."""
    sets = [set(l.tolist()) for l in L]
    out = []
    for t, l in enumerate(L):
        def level(j):
            for g in (32, 16, 8, 4, 2):
                b = (t // g) * g
                if all(j in sets[u] for u in range(b, b + g) if u < len(L)):
                    return g
            return 1
        out.append(np.array(sorted(l, key=lambda j: (-level(j), j))))
    return out


T_, P_, S_ = 0, 0, 0
for w0 in warps:
    L = hier_order(lists_for(w0))
    a, b, k = distinct_per_step(L)
    T_ += a; P_ += b; S_ += k
print('hier distinct per step %.2f, per pair %.3f, steps/warp %.1f' % (T_ / S_, T_ / P_, S_ / len(warps)))
