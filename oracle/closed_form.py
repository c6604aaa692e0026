"""ORACLE — TEST INFRASTRUCTURE ONLY.  Pin P6: closed-form size
of the unpruned dependent-range space of Fig 11.

Without constraints the 15-tuple splits, for fixed (blk_k, dim_vec), into an
"m side" (dim_m, blk_m, dim_m_a, dim_n_a) and an "n side" (dim_n, blk_n,
dim_m_b, dim_n_b):

  N_space = 16 * sum_{dim_vec} nvm(dim_vec) * sum_{blk_k}
              [ sum_{blk_m} m(blk_m) * |A(blk_m, blk_k, dim_vec)| ]
            * [ sum_{blk_n} n(blk_n) * |B(blk_k, blk_n, dim_vec)| ]

where m(blk_m) = #{dim_m <= dim_m_max : dim_m | blk_m} (blk_m runs over the
multiples of dim_m), nvm = 1 if dim_vec == 1 else 2
(PAPER.md:1070-1077), |A| = (RA_m)(RA_n) from PAPER.md:1079-1095, |B| from
PAPER.md:1097-1113, and 16 = 2^4 for tex_a, tex_b, shmem_l1, shmem_banks
(PAPER.md:1115-1118).
"""
from __future__ import annotations

from . import resolve


def n_space(space: dict) -> int:
    s = resolve(space)
    prec = space["precision"]
    dvs = {"D": (1, 2), "S": (1, 4), "C": (1, 2), "Z": (1,)}[prec]   # reading A1
    DMX, DNX, BMX, BNX, BKX = (s["dim_m_max"], s["dim_n_max"], s["blk_m_max"],
                              s["blk_n_max"], s["blk_k_max"])
    ta, tb = s["trans_a"], s["trans_b"]

    def mult(b, dmax):
        return sum(1 for d in range(1, dmax + 1) if b % d == 0)

    m_of = {bm: mult(bm, DMX) for bm in range(1, BMX + 1)}
    n_of = {bn: mult(bn, DNX) for bn in range(1, BNX + 1)}
    total = 0
    for dv in dvs:
        nvm = 1 if dv == 1 else 2
        for bk in range(1, BKX + 1):
            a_side = 0
            for bm in range(1, BMX + 1):
                ram = (bm if ta == 0 else bk) // dv
                ran = bk if ta == 0 else bm
                a_side += m_of[bm] * ram * ran
            b_side = 0
            for bn in range(1, BNX + 1):
                rbm = (bk if tb == 0 else bn) // dv
                rbn = bn if tb == 0 else bk
                b_side += n_of[bn] * rbm * rbn
            total += nvm * a_side * b_side
    return 16 * total
