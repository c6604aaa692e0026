"""Development: per-tile timeline of the three prefix levels from a
BEAST_TILE_TRACE build (scripts/build_variant.sh trace -DBEAST_TILE_TRACE).
Usage: BEAST_LIB_PATH=variants/trace.so python scripts/tile_trace.py [space]"""
import ctypes
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402
from paper_conf_ipps_luszczekgkdd16_b200 import _lib  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "headline"
sp = beast.Space.from_desc(bi.named(name))
n = sp.count()
out = torch.empty((max(n, 1), 2), dtype=torch.uint64, device="cuda")
for _ in range(3):
    beast.beast_enumerate(sp.handle, out)
torch.cuda.synchronize()
buf = np.zeros(3 * 8192 * 5, dtype=np.uint64)
lib = ctypes.CDLL(_lib.LIB_PATH)
assert lib.beast_debug_tile_trace(buf.ctypes.data_as(ctypes.c_void_p)) == 0
tr = buf.reshape(3, 8192, 5).astype(np.int64)
t0 = tr[0][tr[0][:, 0] > 0][:, 0].min()
for lv, nm in enumerate(["L1-L3", "L4", "L5-L7"]):
    t = tr[lv]
    m = t[:, 0] > 0
    t = t[m]
    if not len(t):
        continue
    s, c, l, e = (t[:, i] - t0 for i in range(4))
    print("%s: %d tiles, start %.1f..%.1f us, counted +%.2f us (med), looked back +%.2f us (med, max %.2f), "
          "emitted +%.2f us (med, max %.2f), end of level %.1f us" % (
              nm, len(t), s.min() / 1e3, s.max() / 1e3, np.median(c - s) / 1e3, np.median(l - c) / 1e3,
              (l - c).max() / 1e3, np.median(e - l) / 1e3, (e - l).max() / 1e3, e.max() / 1e3))
    order = np.argsort(s)
    q = np.linspace(0, len(t) - 1, 9).astype(int)
    print("   tile-ordered end times (us):", ["%.1f" % (e[i] / 1e3) for i in q])
    print("   look-back done (us) at tile quantiles:", ["%.1f" % (l[i] / 1e3) for i in q])
    print("   distinct CTAs %d, words max %d" % (len(set(t[:, 4] & 0xffffffff)), (t[:, 4] >> 32).max()))
    idx = np.nonzero(m)[0]
    for i in np.argsort(-e)[:4]:
        print("   late tile %d: start %.2f counted %.2f looked back %.2f emitted %.2f us, words %d" % (
            idx[i], s[i] / 1e3, c[i] / 1e3, l[i] / 1e3, e[i] / 1e3, t[i, 4] >> 32))
for lv in range(3):
    t = tr[lv]
    for k in range(3):
        if t[k, 0] > 0:
            print("level %d tile %d: start %.2f counted %.2f looked back %.2f emitted %.2f us, words %d" % (
                lv, k, (t[k, 0] - t0) / 1e3, (t[k, 1] - t0) / 1e3, (t[k, 2] - t0) / 1e3, (t[k, 3] - t0) / 1e3,
                t[k, 4] >> 32))

# k_tile_eval timeline (last pass): reset the tile counter, run one pass, read
tl = np.zeros(2 * 8192 * 3, dtype=np.uint64)
ct = np.zeros(2 * 1024 * 2, dtype=np.uint64)
lib.beast_debug_eval_trace(tl.ctypes.data_as(ctypes.c_void_p), ct.ctypes.data_as(ctypes.c_void_p))
beast.beast_enumerate(sp.handle, out)
torch.cuda.synchronize()
lib.beast_debug_eval_trace(tl.ctypes.data_as(ctypes.c_void_p), ct.ctypes.data_as(ctypes.c_void_p))
tl = tl.reshape(2, 8192, 3).astype(np.int64)
ct = ct.reshape(2, 1024, 2).astype(np.int64)
for st, nm in ((0, "A"), (1, "B")):
    t = tl[st][tl[st][:, 0] > 0]
    c = ct[st][ct[st][:, 0] > 0]
    if not len(t):
        continue
    base = c[:, 0].min()
    dur = (t[:, 1] - t[:, 0]) / 1e3
    print("k_tile_eval<%s>: CTAs start %.1f..%.1f us, end %.1f..%.1f us; %d tiles, tile time med %.2f max %.2f us, "
          "jobs med %d; first tile start %.1f, last tile end %.1f us" % (
              nm, 0, (c[:, 0].max() - base) / 1e3, (c[:, 1].min() - base) / 1e3, (c[:, 1].max() - base) / 1e3,
              len(t), np.median(dur), dur.max(), np.median(t[:, 2] >> 32), (t[:, 0].min() - base) / 1e3,
              (t[:, 1].max() - base) / 1e3))
