"""ORACLE — TEST INFRASTRUCTURE ONLY.  Pin P5: an independent
analytic counter.

It computes the same statistics as the canonical nest (visits per level L1..L15,
first-failing rejections, survivors) without walking the inner loops L8..L15:
for every prefix that passes Figs 13/14 it counts the valid A-read grids by
enumerating the divisors x of threads_per_block (cant_reshape_a1,
PAPER.md:1370-1372, can only be False when dim_m_a * dim_n_a == T, i.e. for
dim_m_a = x | T, dim_n_a = T / x) and then tests cant_reshape_a2
 on those few candidates; likewise for B
(PAPER.md:1374-1376, 1387-1394).  Loops L1..L6 are vectorised with numpy per
(dim_m, dim_n) pair.  It shares no code and no loop structure with
beast_oracle.c.

The level at which each predicate is charged follows reading A6 (the
canonical hoisted nest): L2 over_max_threads, partial_warps; L4
over_max_regs_per_thread, over_max_regs_per_block, low_occupancy_regs; L5
over_max_shmem, low_occupancy_shmem; L6 low_fmas; L9 a1, a2; L11 b1, b2.
"""
from __future__ import annotations

import numpy as np

from . import resolve


def _dim_vec_values(prec: str):
    # Fig 11 dim_vec, reading A1: D {1,2}, S {1,4},
    # C {1,2}, Z {1}.
    return {"D": (1, 2), "S": (1, 4), "C": (1, 2), "Z": (1,)}[prec]


def _divisors(t: int):
    return [x for x in range(1, t + 1) if t % x == 0]


def _add_shapes(hist: dict, rows, cols, weight) -> None:
    """hist[(rows, cols)] += weight, for parallel arrays."""
    if rows.size == 0:
        return
    key = np.stack([rows, cols], axis=1)
    uk, inv = np.unique(key, axis=0, return_inverse=True)
    w = np.bincount(inv.ravel(), weights=weight.astype(np.float64), minlength=len(uk))
    for (a, b), c in zip(uk.tolist(), w.tolist()):
        if c:
            hist[(a, b)] = hist.get((a, b), 0) + int(round(c))


def count(space: dict, shapes: bool = False) -> dict:
    """Returns dict(visits[15], rejected[12], survivors, prefixes (L7 visits),
    valid_a (number of (prefix, dim_m_a, dim_n_a) passing a1 and a2)).
    shapes=True adds the grid-shape histograms of the L8-L11 loops:
    a_shapes[(RA_m, RA_n)] = number of L7 prefixes whose A-read grid
    (dim_m_a in 1..RA_m, dim_n_a in 1..RA_n) has that shape, and
    b_shapes[(RB_m, RB_n)] = number of valid (prefix, A grid) pairs whose
    B-read grid has that shape -- sum(RA_m * RA_n * count) is
    visits[8] and sum(RB_m * RB_n * count) is visits[10]."""
    a_shapes, b_shapes = {}, {}
    s = resolve(space)
    prec = space["precision"]
    cr = 2 if prec in ("D", "Z") else 1
    cx = 2 if prec in ("C", "Z") else 1
    ta, tb = s["trans_a"], s["trans_b"]
    DMX, DNX, BMX, BNX, BKX = (s["dim_m_max"], s["dim_n_max"], s["blk_m_max"],
                              s["blk_n_max"], s["blk_k_max"])
    V = [0] * 15
    R = [0] * 12
    valid_a = 0
    tuples = 0

    # L1 x L2 as a grid
    dm = np.arange(1, DMX + 1, dtype=np.int64)[:, None]
    dn = np.arange(1, DNX + 1, dtype=np.int64)[None, :]
    T = dm * dn
    V[0] = DMX
    V[1] = DMX * DNX
    over = T > s["max_threads_per_block"]
    partial = (~over) & (T % s["warp_size"] != 0)
    R[0] = int(over.sum())
    R[7] = int(partial.sum())
    ok_pairs = np.argwhere(~over & ~partial)
    bk = np.arange(1, BKX + 1, dtype=np.int64)

    for i, j in ok_pairs:
        dim_m, dim_n = int(i) + 1, int(j) + 1
        t = dim_m * dim_n
        K = BMX // dim_m          # number of blk_m values (L3 trip count)
        Lc = BNX // dim_n         # number of blk_n values (L4 trip count)
        V[2] += K
        V[3] += K * Lc
        if K == 0 or Lc == 0:
            continue
        thr_m = np.arange(1, K + 1, dtype=np.int64)[:, None]
        thr_n = np.arange(1, Lc + 1, dtype=np.int64)[None, :]
        rpt = thr_m * thr_n * cr * cx
        r1 = rpt > s["max_registers_per_thread"]
        rpb = rpt * t
        r2 = ~r1 & (rpb > s["max_regs_per_block"])
        mbr = np.minimum(s["max_registers_per_multi_processor"] // rpb,
                         s["max_blocks_per_multi_processor"])
        r4 = ~r1 & ~r2 & (mbr * t < s["min_threads_per_multi_processor"])
        R[1] += int(r1.sum()); R[2] += int(r2.sum()); R[4] += int(r4.sum())
        keep = ~(r1 | r2 | r4)
        ki, li = np.nonzero(keep)
        if ki.size == 0:
            continue
        tm = (ki + 1).astype(np.int64)[:, None]   # thr_m of each L4 survivor
        tn = (li + 1).astype(np.int64)[:, None]
        blk_m = tm * dim_m
        blk_n = tn * dim_n
        blk_k = bk[None, :]
        V[4] += ki.size * BKX
        spb = blk_k * (blk_m + blk_n) * s["float_size"] * cr * cx
        r3 = spb > s["max_shared_mem_per_block"]
        mbs = np.minimum(s["max_shmem_per_multi_processor"] // spb,
                         s["max_blocks_per_multi_processor"])
        r5 = ~r3 & (mbs * t < s["min_threads_per_multi_processor"])
        R[3] += int(r3.sum()); R[5] += int(r5.sum())
        p5 = ~(r3 | r5)
        # broadcast everything to the (L4 survivor, blk_k) grid and flatten
        # the L5 survivors
        TM = np.broadcast_to(tm, p5.shape)[p5]
        TN = np.broadcast_to(tn, p5.shape)[p5]
        BM = np.broadcast_to(blk_m, p5.shape)[p5]
        BN = np.broadcast_to(blk_n, p5.shape)[p5]
        BK = np.broadcast_to(blk_k, p5.shape)[p5]
        for dv in _dim_vec_values(prec):
            V[5] += BK.size
            lpb = (TM + TN) * BK // dv * t * cx
            fpb = TM * TN * BK * t * cx * cx
            with np.errstate(divide="ignore"):
                ratio = np.where(lpb == 0, -1, fpb // np.where(lpb == 0, 1, lpb))
            r6 = (lpb == 0) | (ratio < s["min_fmas_per_load"])
            R[6] += int(r6.sum())
            ok = ~r6
            nvm = 1 if dv == 1 else 2          # vec_mul trip count
            bm, bn, bkk = BM[ok], BN[ok], BK[ok]
            V[6] += nvm * bm.size
            if bm.size == 0:
                continue
            ram = (bm if ta == 0 else bkk) // dv
            ran = bkk if ta == 0 else bm
            rbm = (bkk if tb == 0 else bn) // dv
            rbn = bn if tb == 0 else bkk
            V[7] += nvm * int(ram.sum())
            V[8] += nvm * int((ram * ran).sum())
            if shapes:
                _add_shapes(a_shapes, ram, ran, np.full(ram.shape, nvm))
            a1h = np.zeros_like(bm)
            na = np.zeros_like(bm)
            b1h = np.zeros_like(bm)
            nb = np.zeros_like(bm)
            for x in _divisors(t):
                y = t // x
                a1 = (x <= ram) & (y <= ran)
                a1h += a1
                if ta == 0:
                    a2ok = (bm % (x * dv) == 0) & (bkk % y == 0)
                else:
                    a2ok = (bkk % (x * dv) == 0) & (bm % y == 0)
                na += a1 & a2ok
                b1 = (x <= rbm) & (y <= rbn)
                b1h += b1
                if tb == 0:
                    b2ok = (bkk % (x * dv) == 0) & (bn % y == 0)
                else:
                    b2ok = (bn % (x * dv) == 0) & (bkk % y == 0)
                nb += b1 & b2ok
            R[8] += nvm * int((ram * ran - a1h).sum())
            R[10] += nvm * int((a1h - na).sum())
            V[9] += nvm * int((na * rbm).sum())
            V[10] += nvm * int((na * rbm * rbn).sum())
            R[9] += nvm * int((na * (rbm * rbn - b1h)).sum())
            R[11] += nvm * int((na * (b1h - nb)).sum())
            valid_a += nvm * int(na.sum())
            if shapes:
                _add_shapes(b_shapes, rbm, rbn, nvm * na)
            tuples += nvm * int((na * nb).sum())
    V[11] = 2 * tuples
    V[12] = 4 * tuples
    V[13] = 8 * tuples
    V[14] = 16 * tuples
    out = dict(visits=V, rejected=R, survivors=V[14], prefixes=V[6], valid_a=valid_a)
    if shapes:
        out.update(a_shapes=a_shapes, b_shapes=b_shapes)
    return out
