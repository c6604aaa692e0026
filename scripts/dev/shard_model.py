"""Offline check of the shard work estimate (ScanL4Work): per L4 survivor,
the fitted stage-time model from the exact per-prefix quantities
of the analytic counter's enumeration, against the library's closed-form
estimate re-implemented here; prints the per-shard model cost of the split
each one induces.  Usage: python scripts/dev/shard_model.py [workload] [world]"""
import math
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import beast_inputs as bi  # noqa: E402
import oracle  # noqa: E402

W = dict(FA=0.0264e-9, P=0.0205e-6, CA=0.0096e-6, FB=0.0286e-9, VA=0.0135e-6, TU=0.0643e-6)
RC, CC, PC, VC = 0, 364, 776, 472


def divisors(t):
    return [x for x in range(1, t + 1) if t % x == 0]


def per_l4(space):
    s = oracle.resolve(space)
    prec = space["precision"]
    cr = 2 if prec in ("D", "Z") else 1
    cx = 2 if prec in ("C", "Z") else 1
    ta, tb = s["trans_a"], s["trans_b"]
    DMX, DNX, BMX, BNX, BKX = (s["dim_m_max"], s["dim_n_max"], s["blk_m_max"], s["blk_n_max"], s["blk_k_max"])
    dvs = {"D": (1, 2), "S": (1, 4), "C": (1, 2), "Z": (1,)}[prec]
    true_cost, est, comp, ecomp = [], [], [], []
    bk = np.arange(1, BKX + 1, dtype=np.int64)
    for dim_m in range(1, DMX + 1):
        for dim_n in range(1, DNX + 1):
            T = dim_m * dim_n
            if T > s["max_threads_per_block"] or T % s["warp_size"]:
                continue
            K, Lc = BMX // dim_m, BNX // dim_n
            for thr_m in range(1, K + 1):
                for thr_n in range(1, Lc + 1):
                    rpt = thr_m * thr_n * cr * cx
                    if rpt > s["max_registers_per_thread"]:
                        continue
                    rpb = rpt * T
                    if rpb > s["max_regs_per_block"]:
                        continue
                    if min(s["max_registers_per_multi_processor"] // rpb, s["max_blocks_per_multi_processor"]) * T \
                            < s["min_threads_per_multi_processor"]:
                        continue
                    bm, bn = thr_m * dim_m, thr_n * dim_n
                    spb = bk * (bm + bn) * s["float_size"] * cr * cx
                    ok5 = (spb <= s["max_shared_mem_per_block"]) & \
                          (np.minimum(s["max_shmem_per_multi_processor"] // spb, s["max_blocks_per_multi_processor"]) * T
                           >= s["min_threads_per_multi_processor"])
                    t = int(ok5.sum())     # passing blk_k are 1..t
                    c = 0.0
                    e = 0
                    cc = np.zeros(6)
                    ec = np.zeros(4)
                    for dv in dvs:
                        mult = 1 if dv == 1 else 2
                        k = bk[:t]
                        lpb = (thr_m + thr_n) * k // dv * T * cx
                        fpb = thr_m * thr_n * k * T * cx * cx
                        ok6 = (lpb != 0) & (fpb // np.where(lpb == 0, 1, lpb) >= s["min_fmas_per_load"])
                        kk = k[ok6]
                        ram = (bm if ta == 0 else kk) // dv
                        ran = kk if ta == 0 else bm
                        ram = np.broadcast_to(ram, kk.shape)
                        ran = np.broadcast_to(ran, kk.shape)
                        S, L = np.minimum(ram, ran), np.maximum(ram, ran)
                        FA = (S * 16 * ((L + 15) // 16)).sum()
                        a1 = np.zeros(kk.shape, np.int64)
                        na = np.zeros(kk.shape, np.int64)
                        nb = np.zeros(kk.shape, np.int64)
                        rbm = (kk if tb == 0 else bn) // dv
                        rbn = bn if tb == 0 else kk
                        rbm = np.broadcast_to(rbm, kk.shape)
                        rbn = np.broadcast_to(rbn, kk.shape)
                        for x in divisors(T):
                            y = T // x
                            a1 += (x <= ram) & (y <= ran)
                            a2ok = ((bm % (x * dv) == 0) & (kk % y == 0)) if ta == 0 else \
                                   ((kk % (x * dv) == 0) & (bm % y == 0))
                            na += (x <= ram) & (y <= ran) & a2ok
                            b2ok = ((kk % (x * dv) == 0) & (bn % y == 0)) if tb == 0 else \
                                   ((bn % (x * dv) == 0) & (kk % y == 0))
                            nb += (x <= rbm) & (y <= rbn) & b2ok
                        SB, LB = np.minimum(rbm, rbn), np.maximum(rbm, rbn)
                        FB = (na * SB * 16 * ((LB + 15) // 16)).sum()
                        c += mult * (W["FA"] * FA + W["P"] * kk.size + W["CA"] * a1.sum() + W["FB"] * FB +
                                     W["VA"] * na.sum() + W["TU"] * (na * nb).sum())
                        cc += mult * np.array([FA, kk.size, a1.sum(), FB, na.sum(), (na * nb).sum()], dtype=np.float64)
                        A_, lpt_ = thr_m * thr_n * cx, thr_m + thr_n
                        mf = s["min_fmas_per_load"]
                        if mf == 0 or A_ * dv >= mf * lpt_:
                            k0 = -(-dv // lpt_)
                            p1 = np.array(est_parts(t, bm, bn, T, dv, int(math.log2(dv)), ta, tb), dtype=np.float64)
                            p0 = np.array(est_parts(k0 - 1, bm, bn, T, dv, int(math.log2(dv)), ta, tb), dtype=np.float64) if k0 > 1 else 0
                            ec += mult * (p1 - p0)

                    true_cost.append(c)
                    est.append(ec[0] + ec[1] + CC * ec[2] + PC * ec[3] + 1)
                    comp.append(cc)
                    ecomp.append(ec)
    return np.array(true_cost), np.array(est, dtype=np.float64), np.array(comp), np.array(ecomp)


def grid_cost1(j, M):
    if j == 0 or M == 0:
        return 0
    S, L = min(j, M), max(j, M)
    return S * (16 * ((L + 15) >> 4) + RC)


def est_side(t, bm, bn, T, dv, sh, ta, tb):
    c, b, a1, p = est_parts(t, bm, bn, T, dv, sh, ta, tb)
    return c + b + CC * a1 + PC * p


def est_parts(t, bm, bn, T, dv, sh, ta, tb):
    c = sum(grid_cost1(k if ta == 0 else k >> sh, (bm >> sh) if ta == 0 else bm) for k in range(1, t + 1))
    b = 0
    g = 0 if t == 0 else (math.gcd(T, bm >> sh) if (ta == 0 and (bm & (dv - 1)) == 0) else
                          (math.gcd(T, bm) if ta else 0))
    for x in (divisors(g) if g else []):
        step = T // x if ta == 0 else (T // x) * dv
        J = t // step
        sj = step * (J * (J + 1) // 2)
        b += bn * (sj >> sh) if tb == 0 else (bn >> sh) * sj
        b += VC * J
    a1 = 0
    for x in divisors(T):
        need = (T // x if x <= (bm >> sh) else t + 1) if ta == 0 else (x * dv if T // x <= bm else t + 1)
        if need <= t:
            a1 += t - need + 1
    return c, b, a1, t


def split(weights, world):
    cum = np.concatenate([[0], np.cumsum(weights)])
    Wt = cum[-1]
    bounds = [0]
    for r in range(1, world):
        bounds.append(int(np.searchsorted(cum, Wt * r / world, side="left")))
    bounds.append(len(weights))
    return bounds


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "b200_S"
    world = int(sys.argv[2]) if len(sys.argv) > 2 else 8
    tc, es, comp, ecomp = per_l4(bi.named(name))
    print(name, "L4 survivors", len(tc), "model total %.3f ms" % tc.sum())
    for label, w in (("estimate", es), ("perfect", tc)):
        b = split(w, world)
        per = [tc[b[r]:b[r + 1]].sum() for r in range(world)]
        print("%-9s split: shard model ms %s  balance %.3f" % (label, " ".join("%.3f" % x for x in per),
                                                             np.mean(per) / max(per)))
    # which component of the estimate is off: correlation by dim_m decile
    q = np.array_split(np.arange(len(tc)), 10)
    names = ["FA", "P", "CA", "FB", "VA", "TU"]
    for j, nm in enumerate(names):
        print("model %-3s by decile:" % nm, " ".join("%.3g" % comp[i, j].sum() for i in q))
    for j, nm in enumerate(["A est", "B est", "a1 est", "t est"]):
        print("%-9s by decile:" % nm, " ".join("%.3g" % ecomp[i, j].sum() for i in q))
    print("estimate / model share by decile of the L4 list:", " ".join("%.2f" % (es[i].sum() / es.sum() / (tc[i].sum() / tc.sum())) for i in q))


if __name__ == "__main__":
    main()
