"""SURVEY 8(f) NEXT 4 / PAPER.md §6 (ICA for bounding boxes, "a bounding box can also be approximated
into 2 cylinders"): would a box-based outer cone cull the 256-voxel Morton bricks better than their
bounding sphere?  For every brick of a model (Morton order as the library sorts) and a few pivots, the
half-angle of three exact outer bounds on the directions in which the tool can touch the brick:

  sphere   asin((Reff + r) / D)                     (the library's test; r = half-diagonal of the AABB)
  box      asin(Reff / Dmin) + beta                 (beta = the AABB's angular radius seen from the pivot,
                                                     max over its 8 corners; Dmin = distance to the AABB)
  capsule  asin((Reff + rho) / Dseg) + beta_seg     (the circumscribed cylinder of the AABB along its
                                                     longest axis, bounded by segment + ball rho)

Reff = the radius of the tool cylinders within reach (tip/shank 6.35; 20 beyond the shank).  Prints
the mean half-angles and how often each box-type bound is tighter than the sphere.
    python tools/box_ica_study.py C2 [pivots]
"""
import math
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402


def spread3(v):
    x = v.astype(np.uint64) & np.uint64(0x1fffff)
    for s, m in ((32, 0x1f00000000ffff), (16, 0x1f0000ff0000ff), (8, 0x100f00f00f00f00f), (4, 0x10c30c30c30c30c3),
                 (2, 0x1249249249249249)):
        x = (x | (x << np.uint64(s))) & np.uint64(m)
    return x


def main(name, npiv=6):
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    lo, hi = C.min(0), C.max(0)
    sc = 2097151.0 / max(float((hi - lo).max()), 1e-30)
    q = np.clip((C - lo) * sc, 0, 2097151).astype(np.uint32)
    key = spread3(q[:, 0]) | (spread3(q[:, 1]) << np.uint64(1)) | (spread3(q[:, 2]) << np.uint64(2))
    o = np.argsort(key, kind="stable")
    C, H = C[o].astype(np.float64), H[o].astype(np.float64)
    nb = len(H) // 256
    Cb = C[: nb * 256].reshape(nb, 256, 3)
    Hb = H[: nb * 256].reshape(nb, 256, 1)
    bmin, bmax = (Cb - Hb).min(1), (Cb + Hb).max(1)
    cen, half = 0.5 * (bmin + bmax), 0.5 * (bmax - bmin)
    r = np.linalg.norm(half, axis=1)
    ext = np.sort(half, axis=1)
    ax = np.argmax(half, axis=1)
    print(f"{name}: {nb} bricks; AABB half extents (sorted) median {np.median(ext, 0).round(3)} mm, "
          f"longest / shortest median {np.median(ext[:, 2] / np.maximum(ext[:, 0], 1e-9)):.2f}")
    tot = {"sphere": [], "box": [], "capsule": []}
    better_box = better_cap = 0
    n_all = 0
    for p in cfg.pivots(npiv).astype(np.float64):
        v = cen - p
        D = np.linalg.norm(v, axis=1)
        keep = D > r * 1.01
        v, D, rr, hf, c0, a_ = v[keep], D[keep], r[keep], half[keep], cen[keep], ax[keep]
        reach = D + rr
        Reff = np.where(reach >= 25.4 + 76.2, 20.0, 6.35)
        sph = np.arcsin(np.minimum(1.0, (Reff + rr) / D))
        u = v / D[:, None]
        beta = np.zeros_like(D)
        for k in range(8):
            s = np.array([1 if k & 1 else -1, 1 if k & 2 else -1, 1 if k & 4 else -1], np.float64)
            w = v + s * hf
            cosang = np.clip((w * u).sum(1) / np.linalg.norm(w, axis=1), -1, 1)
            beta = np.maximum(beta, np.arccos(cosang))
        dmin = np.linalg.norm(np.maximum(np.abs(v) - hf, 0.0), axis=1)
        box = np.arcsin(np.minimum(1.0, Reff / np.maximum(dmin, 1e-9))) + beta
        # capsule: segment along the longest axis, radius = half-diagonal of the cross-section
        e = np.zeros_like(v)
        e[np.arange(len(v)), a_] = hf[np.arange(len(v)), a_]
        rho = np.sqrt(np.maximum((hf ** 2).sum(1) - (e ** 2).sum(1), 0.0))
        bseg = np.zeros_like(D)
        for sgn in (-1.0, 1.0):
            w = v + sgn * e
            bseg = np.maximum(bseg, np.arccos(np.clip((w * u).sum(1) / np.linalg.norm(w, axis=1), -1, 1)))
        dseg = np.maximum(D - np.linalg.norm(e, axis=1), 1e-9)
        cap = np.arcsin(np.minimum(1.0, (Reff + rho) / dseg)) + bseg
        tot["sphere"].append(sph)
        tot["box"].append(box)
        tot["capsule"].append(cap)
        better_box += int((box < sph).sum())
        better_cap += int((cap < sph).sum())
        n_all += len(D)
    for k in tot:
        a = np.concatenate(tot[k])
        print(f"  {k:8s} mean half-angle {np.degrees(a.mean()):6.2f} deg, median {np.degrees(np.median(a)):6.2f}")
    both = np.minimum(np.concatenate(tot["sphere"]), np.minimum(np.concatenate(tot["box"]), np.concatenate(tot["capsule"])))
    s_all = np.concatenate(tot["sphere"])
    print(f"  box tighter than sphere for {100 * better_box / n_all:.1f} % of (brick, pivot) pairs, capsule for "
          f"{100 * better_cap / n_all:.1f} %; the best of the three narrows the mean cone by "
          f"{100 * (1 - both.mean() / s_all.mean()):.2f} % (solid angle ~ angle^2: "
          f"{100 * (1 - (both ** 2).mean() / (s_all ** 2).mean()):.2f} %)")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "C2", int(sys.argv[2]) if len(sys.argv) > 2 else 6)
