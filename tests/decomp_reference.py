"""Host (numpy / torch-CPU) reference of the SFC decomposition's selection logic
 -- test infrastructure: the CPU gloo tests drive it through the
real collectives of paper_conf_sc_simsekpc24_b200.decomp.Comm, and the GPU
tests compare libsph's device routing (include/sph.h "SFC decomposition on the
device") with it element by element."""
from __future__ import annotations

import numpy as np
import torch

HIST_BITS = 15


def red7(x, y, z, h):
    """(-min x, -min y, -min z, max x, max y, max z, max h); -inf when empty."""
    if x.size == 0:
        return np.full(7, -np.inf)
    return np.array([-x.min(), -y.min(), -z.min(), x.max(), y.max(), z.max(), h.max()])


def key_box(red, params):
    """The box of the keys: configured on periodic axes, [-red[a], red[3+a]] on open ones."""
    lo = np.array([params.box_min[a] if params.periodic[a] else -red[a] for a in range(3)])
    hi = np.array([params.box_max[a] if params.periodic[a] else red[3 + a] for a in range(3)])
    return lo, hi


def splits_from_hist(hist, world):
    """s_0 = 0, s_world = nb; s_r = first bin whose inclusive prefix count exceeds
    floor(total r / world) (nb when never exceeded)."""
    hist = np.asarray(hist, dtype=np.int64)
    nb = hist.size
    cum = np.cumsum(hist)
    total = int(cum[-1]) if nb else 0
    s = [0]
    for r in range(1, world):
        t = total * r // world
        s.append(int(np.searchsorted(cum, t, side="right")) if t < total else nb)
    s.append(nb)
    return np.array(s, dtype=np.int64)


def owners(keys, splits, bits=HIST_BITS):
    b = (np.asarray(keys, dtype=np.uint64) >> np.uint64(63 - bits)).astype(np.int64)
    return np.searchsorted(splits, b, side="right") - 1


def _compact3(v):
    v = v & np.uint64(0x1249249249249249)
    for sh, m in ((2, 0x10c30c30c30c30c3), (4, 0x100f00f00f00f00f), (8, 0x1f0000ff0000ff),
                  (16, 0x1f00000000ffff), (32, 0x1fffff)):
        v = (v ^ (v >> np.uint64(sh))) & np.uint64(m)
    return v.astype(np.int64)


def _spread3(v):
    v = np.asarray(v, dtype=np.uint64) & np.uint64(0x1fffff)
    for sh, m in ((32, 0x1f00000000ffff), (16, 0x1f0000ff0000ff), (8, 0x100f00f00f00f00f),
                  (4, 0x10c30c30c30c30c3), (2, 0x1249249249249249)):
        v = (v | (v << np.uint64(sh))) & np.uint64(m)
    return v


def ghost_level(lo, hi, hmax):
    L = 21
    while L > 0:
        side = (hi - lo) / float(1 << L)
        if np.all(side >= 2.0 * hmax * (1.0 + 1e-9)):
            break
        L -= 1
    return L


def ghost_masks_cells(keys, lo, hi, hmax, periodic, splits, rank, world, bits=HIST_BITS):
    """Bit r of mask[i]: a rank r != `rank` owns a key of one of the 27 level-L cells
    around particle i's (L: cell side >= 2 h_max; periodic wrap, open faces clipped)."""
    keys = np.asarray(keys, dtype=np.uint64)
    L = ghost_level(lo, hi, hmax)
    lb = bits // 3
    nside = 1 << L
    c = np.stack([_compact3(keys >> np.uint64(2)), _compact3(keys >> np.uint64(1)), _compact3(keys)], 1) >> (21 - L)
    mask = np.zeros(keys.size, dtype=np.uint64)
    for o in range(27):
        off = np.array([o // 9 - 1, (o // 3) % 3 - 1, o % 3 - 1])
        u = c + off
        ok = np.ones(keys.size, dtype=bool)
        for a in range(3):
            out = (u[:, a] < 0) | (u[:, a] >= nside)
            if periodic[a]:
                u[:, a] = np.mod(u[:, a], nside)
            else:
                ok &= ~out
        ck = (_spread3(u[:, 0]) << np.uint64(2)) | (_spread3(u[:, 1]) << np.uint64(1)) | _spread3(u[:, 2])
        if L >= lb:
            b0 = b1 = (ck >> np.uint64(3 * (L - lb))).astype(np.int64)
        else:
            b0 = (ck << np.uint64(3 * (lb - L))).astype(np.int64)
            b1 = ((ck + np.uint64(1)) << np.uint64(3 * (lb - L))).astype(np.int64) - 1
        r0 = np.searchsorted(splits, b0, side="right") - 1
        r1 = np.searchsorted(splits, b1, side="right") - 1
        for r in range(world):
            sel = ok & (r0 <= r) & (r <= r1)
            mask[sel] |= np.uint64(1 << r)
    mask &= ~np.uint64(1 << rank)
    return mask


# ---- the AABB selection of the legacy sph_select_ghosts (kept in the ABI)
def box_distance(x, lo, hi, box_len, periodic):
    """Minimum-image distance of points x [n,3] to the axis-aligned box [lo, hi]."""
    d2 = torch.zeros(x.shape[0], dtype=x.dtype, device=x.device)
    for a in range(3):
        if periodic[a]:
            best = None
            for k in (-1.0, 0.0, 1.0):
                xa = x[:, a] + k * box_len[a]
                da = torch.clamp(torch.maximum(lo[a] - xa, xa - hi[a]), min=0.0)
                best = da if best is None else torch.minimum(best, da)
        else:
            best = torch.clamp(torch.maximum(lo[a] - x[:, a], x[:, a] - hi[a]), min=0.0)
        d2 = d2 + best * best
    return torch.sqrt(d2)


def ghost_masks_boxes(x, boxes, rank, radius, box_len, periodic):
    """masks[r]: particles within `radius` of rank r's box (r != rank)."""
    out = []
    for r in range(boxes.shape[0]):
        if r == rank or not torch.isfinite(boxes[r]).all():
            out.append(torch.zeros(x.shape[0], dtype=torch.bool, device=x.device))
            continue
        out.append(box_distance(x, boxes[r, 0], boxes[r, 1], box_len, periodic) < radius)
    return out
