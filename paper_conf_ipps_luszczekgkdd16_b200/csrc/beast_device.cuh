// beast_device.cuh — device-side building blocks of the BEAST enumerator.
//
// Shared by the kernels in beast.cu only (the CPU oracle shares nothing with
// this file).  Citations "P:<line>" are lines of PAPER.md.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace beast {

// ---------------------------------------------------------------- constants
constexpr int kMaxBound = 4095;            // 12-bit packed record fields
constexpr int kMaxBuckets = kMaxBound + 1; // one flattener bucket per loop length L
constexpr int kWarp = 32;
constexpr uint32_t kFull = 0xffffffffu;

// Resolved space, passed by value to every kernel (constant bank).
struct SpaceParams {
    // Fig 8 and Fig 9, resolved
    int64_t max_threads_per_block;
    int64_t max_shared_mem_per_block;
    int64_t warp_size;
    int64_t max_regs_per_block;
    int64_t max_registers_per_multi_processor;
    int64_t max_shmem_per_multi_processor;
    int64_t float_size;
    int64_t max_blocks_per_multi_processor;
    int64_t max_registers_per_thread;
    // Fig 12 factors: cr = 2 for double, cx = 2 for complex
    int64_t cr, cx;
    // Fig 10
    int32_t trans_a, trans_b;
    // Fig 14
    int64_t min_threads_per_multi_processor;
    int64_t min_fmas_per_load;
    // Fig 11 upper limits (reading A9)
    int32_t dim_m_max, dim_n_max, blk_m_max, blk_n_max, blk_k_max;
    // dim_vec set (reading A1): dv[0] = 1, dv[1] in {2, 4} or none
    int32_t n_dv;
    int32_t dv1;
    int32_t log2_dv1;
};

// ------------------------------------------------------------ packed words
// Prefix word = the "hi" half of a survivor record (include/beast.h):
//   [63:52] dim_m [51:40] dim_n [39:28] blk_m [27:16] blk_n [15:4] blk_k
//   [3:1] dim_vec [0] vec_mul
__host__ __device__ __forceinline__ uint32_t hi_dim_m(uint64_t h) { return (uint32_t)(h >> 52) & 0xfff; }
__host__ __device__ __forceinline__ uint32_t hi_dim_n(uint64_t h) { return (uint32_t)(h >> 40) & 0xfff; }
__host__ __device__ __forceinline__ uint32_t hi_blk_m(uint64_t h) { return (uint32_t)(h >> 28) & 0xfff; }
__host__ __device__ __forceinline__ uint32_t hi_blk_n(uint64_t h) { return (uint32_t)(h >> 16) & 0xfff; }
__host__ __device__ __forceinline__ uint32_t hi_blk_k(uint64_t h) { return (uint32_t)(h >> 4) & 0xfff; }
__host__ __device__ __forceinline__ uint32_t hi_dim_vec(uint64_t h) { return (uint32_t)(h >> 1) & 0x7; }

// Flattener job info word (one per job = L7 prefix for the A grids, valid A
// grid for the B grids):  [63:32] job id  [31:16] threads_per_block
//   [13:1] S (rows = length of the short axis)  [0] short axis is the "m" one
__device__ __forceinline__ uint64_t make_info(uint32_t id, uint32_t T, uint32_t S, uint32_t short_m) {
    return ((uint64_t)id << 32) | ((uint64_t)T << 16) | ((uint64_t)S << 1) | short_m;
}
__device__ __forceinline__ uint32_t info_id(uint64_t w) { return (uint32_t)(w >> 32); }
__device__ __forceinline__ uint32_t info_T(uint64_t w) { return (uint32_t)(w >> 16) & 0xffff; }
__device__ __forceinline__ uint32_t info_S(uint64_t w) { return (uint32_t)(w >> 1) & 0x1fff; }
__device__ __forceinline__ uint32_t info_short_m(uint64_t w) { return (uint32_t)w & 1; }

// Valid-grid word: [63:24] owner id (prefix index or valid-A index)
//   [23:12] first coordinate (dim_m_a / dim_m_b) [11:0] second (dim_n_a / dim_n_b)
__device__ __forceinline__ uint64_t make_grid(uint64_t owner, uint32_t m, uint32_t n) {
    return (owner << 24) | ((uint64_t)m << 12) | n;
}
__device__ __forceinline__ uint64_t grid_owner(uint64_t g) { return g >> 24; }
__device__ __forceinline__ uint32_t grid_m(uint64_t g) { return (uint32_t)(g >> 12) & 0xfff; }
__device__ __forceinline__ uint32_t grid_n(uint64_t g) { return (uint32_t)g & 0xfff; }

// ------------------------------------------------------------ warp helpers
__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

// splitmix64 finaliser (the digests of include/beast.h)
__device__ __forceinline__ uint64_t sm64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__device__ __forceinline__ uint64_t ld_volatile_u64(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ void st_volatile_u64(uint64_t *p, uint64_t v) {
    asm volatile("st.volatile.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Exclusive scan of one u32 per thread over a CTA of NT threads.
// Returns the thread's exclusive prefix; *total receives the CTA sum.
template <int NT>
__device__ __forceinline__ uint32_t cta_exclusive_scan(uint32_t v, uint32_t *smem_warp, uint32_t *total) {
    const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(kFull, x, o);
        if ((int)lane >= o) x += y;
    }
    if (lane == 31) smem_warp[warp] = x;
    __syncthreads();
    if (warp == 0) {
        uint32_t w = lane < NT / 32 ? smem_warp[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(kFull, w, o);
            if ((int)lane >= o) w += y;
        }
        if (lane < NT / 32) smem_warp[lane] = w;
    }
    __syncthreads();
    const uint32_t warp_excl = warp ? smem_warp[warp - 1] : 0;
    *total = smem_warp[NT / 32 - 1];
    __syncthreads();
    return warp_excl + x - v;
}

// Same for u64.
template <int NT>
__device__ __forceinline__ uint64_t cta_exclusive_scan64(uint64_t v, uint64_t *smem_warp, uint64_t *total) {
    const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
    uint64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(kFull, x, o);
        if ((int)lane >= o) x += y;
    }
    if (lane == 31) smem_warp[warp] = x;
    __syncthreads();
    if (warp == 0) {
        uint64_t w = lane < NT / 32 ? smem_warp[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint64_t y = __shfl_up_sync(kFull, w, o);
            if ((int)lane >= o) w += y;
        }
        if (lane < NT / 32) smem_warp[lane] = w;
    }
    __syncthreads();
    const uint64_t warp_excl = warp ? smem_warp[warp - 1] : 0;
    *total = smem_warp[NT / 32 - 1];
    __syncthreads();
    return warp_excl + x - v;
}

// --------------------------------------------------- the hot inner loop
// cant_reshape_a1 / b1: "dim_m_x * dim_n_x != threads_per_block".
// A grid row holds its short-axis coordinate s fixed while the long-axis
// coordinate j runs 1..L, so the row's points are the products s*j, j <= L.
//
// Each lane evaluates TWO rows s1 < s2 of the same job at once, one per
// 16-bit half: with Sp = s1 | s2 << 16 and C = (2^16 - T) * 0x10001, the
// word Sp*j + C (mod 2^32) holds (s1*j - T) mod 2^16 in its low half and
// (s2*j - T) mod 2^16 in its high half whenever s1*j < T (no carry reaches
// the high half) — in particular whenever s2*j == T, because s1 < s2.  So a
// point with s*j == T always leaves a zero half (no false negatives); a zero
// half can also come from s*j == T (mod 2^16) with s*j != T, which the exact
// check after the loop rejects.  One IMAD forms a pair of points, and ptxas
// fuses two min.u16x2 into one VIMNMX3.U16x2 folding two pairs into the
// running per-half minimum; the other half of a block uses the packed
// add-and-min VIADDMNMX.U16x2.  With KI of the 16 pairs on the IMAD path,
// 32 points cost KI IMAD (FMA-heavy pipe) + KI/2 VIMNMX3 + (16 - KI)
// VIADDMNMX (ALU pipe).  In isolation KI = 8 is fastest
// (scripts/micro/scan.cu), but the rest of k_eval is ALU-heavy (ncu r01e:
// ALU 66% vs FMA 27% of peak), so the kernel is fastest at KI = 12 (A/B on
// the B200, headline and SGEMM-B200); the block loop is unrolled twice (the
// default 16/8/4/1 cascade costs more than it saves at ~5 blocks per row).
#ifndef BEAST_SCAN_KI
#define BEAST_SCAN_KI 12
#endif
#ifndef BEAST_SCAN_UNROLL
#define BEAST_SCAN_UNROLL 4
#endif
#define BEAST_PRAGMA(x) _Pragma(#x)
#define BEAST_UNROLL(n) BEAST_PRAGMA(unroll n)
template <int KI>
__device__ __forceinline__ void eval16pp(uint32_t &acc, uint32_t &acc2, uint32_t Cb, uint32_t Sp,
                                         const uint32_t (&M)[16 - KI + (KI == 16)]) {
    // j = 1..KI: IMAD products folded pairwise by VIMNMX3 (FMA-heavy + ALU
    // pipes); j = KI+1..16: one packed add-and-min per pair of points,
    // min(acc, Cb + M[j-KI-1]) per 16-bit half (VIADDMNMX.U16x2, ALU pipe),
    // with the loop invariants M[i] = (KI + 1 + i) * Sp.  The halves of Cb + M
    // are formed mod 2^16 without a carry between them; the high half of Cb
    // itself carries no low-half carry whenever the high row has a true
    // match (see scan_rows), so both forms leave a zero exactly where the
    // IMAD form does.
#pragma unroll
    for (int j = 1; j <= KI; j += 2)
        asm volatile("{\n\t.reg .b32 t0, t1;\n\t"
                     "mad.lo.u32 t0, %2, %3, %1;\n\t mad.lo.u32 t1, %2, %4, %1;\n\t"
                     "min.u16x2 %0, %0, t0;\n\t min.u16x2 %0, %0, t1;\n\t}"
                     : "+r"(acc)
                     : "r"(Cb), "r"(Sp), "r"((uint32_t)j), "r"((uint32_t)(j + 1)));
#pragma unroll
    for (int i = 0; i < 16 - KI; ++i)
        asm volatile("{\n\t.reg .b32 t;\n\tadd.u16x2 t, %1, %2;\n\tmin.u16x2 %0, %0, t;\n\t}"
                     : "+r"(acc2) : "r"(Cb), "r"(M[i]));
}

__device__ __forceinline__ uint32_t vmin_u16x2(uint32_t a, uint32_t b) {
    uint32_t r;
    asm("min.u16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
    return r;
}

// Zero halves of the packed scan of a row pair: rows s1 < s2 (s2 == 0:
// single row) of one job against T over j = 1..L (T <= 65535, s, L <= 4095).
// The loop runs NB >= ceil(L/16) blocks (NB is uniform across the warp);
// products past L are computed but a match there is rejected by the exact
// check (t <= L).  Returns the running per-half minimum: a zero half marks a
// candidate row.
__device__ __forceinline__ uint32_t scan_rows(uint32_t s1, uint32_t s2, uint32_t T, uint32_t NB) {
    const uint32_t Sp = s1 | (s2 << 16);
    uint32_t Cb = (0x10000u - T) * 0x10001u;
    asm volatile("" : "+r"(Cb));             // keep C as one register (no per-block re-derivation)
    const uint32_t step = Sp << 4;           // Sp * 16: advance both rows by 16 points
    constexpr int KI = BEAST_SCAN_KI;
    uint32_t M[16 - KI + (KI == 16)];
#pragma unroll
    for (int i = 0; i < 16 - KI; ++i) M[i] = Sp * (uint32_t)(KI + 1 + i);   // halves exact: 16 * 4095 < 2^16
    uint32_t acc = 0xffffffffu, acc2 = 0xffffffffu;   // two chains: IMAD/VIMNMX3 and VIADDMNMX
    BEAST_UNROLL(BEAST_SCAN_UNROLL)
    for (uint32_t b = 0; b < NB; ++b) {
        eval16pp<KI>(acc, acc2, Cb, Sp, M);
        Cb += step;
    }
    return vmin_u16x2(acc, acc2);
}

// The same scan in the instrumented build: `blocks` is incremented inside
// the loop body, once per executed 16-point iteration b < nb_own
// (beast_stats.formed; nb_own = ceil(L / 16) of the lane's own rows, which is
// below the warp's NB when the warp's rows come from jobs of different
// lengths).  (A separate function, so the timed kernels keep scan_rows'
// exact code.)
__device__ __forceinline__ uint32_t scan_rows_counted(uint32_t s1, uint32_t s2, uint32_t T, uint32_t NB,
                                                      uint32_t nb_own, uint32_t &blocks) {
    const uint32_t Sp = s1 | (s2 << 16);
    uint32_t Cb = (0x10000u - T) * 0x10001u;
    asm volatile("" : "+r"(Cb));
    const uint32_t step = Sp << 4;
    constexpr int KI = BEAST_SCAN_KI;
    uint32_t M[16 - KI + (KI == 16)];
#pragma unroll
    for (int i = 0; i < 16 - KI; ++i) M[i] = Sp * (uint32_t)(KI + 1 + i);
    uint32_t acc = 0xffffffffu, acc2 = 0xffffffffu;
    BEAST_UNROLL(BEAST_SCAN_UNROLL)
    for (uint32_t b = 0; b < NB; ++b) {
        eval16pp<KI>(acc, acc2, Cb, Sp, M);
        Cb += step;
        asm volatile("{\n\t.reg .pred p;\n\tsetp.lt.u32 p, %1, %2;\n\t@p add.u32 %0, %0, 1;\n\t}"
                     : "+r"(blocks) : "r"(b), "r"(nb_own));   // counted where the block runs
    }
    return vmin_u16x2(acc, acc2);
}

// fp32 reciprocal (MUFU.RCP, flush-to-zero: operands are integers >= 1 or 0)
__device__ __forceinline__ float rcp_ftz(float x) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}

// Exact, branch-free check of one candidate row s (0 = idle half) of a job
// with threads_per_block T and grid sides S (short) x L (long), after the
// packed scan left `zero` (the row's half of the running minimum is 0):
//   *t    = T / s when s * t == T and t <= L (the a1/b1 pass), else garbage
//   a1    = the scan found the row's zero and s * t == T, t <= L
//   valid = a1 and the divisibility predicate is False: xdiv, s | S, t | L.
// Quotients are formed with the fp32 reciprocal: for a < 2^16 and d < 2^16
// the relative error of a * rcp(d) is ~2^-22, far below 1/2 of the quotient's
// unit, so rounding gives a / d exactly whenever d divides a, and the integer
// products decide (a wrong quotient can only fail a product check).
struct RowCheck { uint32_t t; bool a1, valid; };
__device__ __forceinline__ RowCheck check_row(uint32_t s, bool zero, uint32_t T, uint32_t S, uint32_t L,
                                              float fT, float fS, float fL, bool xdiv) {
    const float r = rcp_ftz((float)s);
    RowCheck c;
    c.t = __float2uint_rn(fT * r);
    const uint32_t q = __float2uint_rn(fS * r);
    const uint32_t u = __float2uint_rn(fL * rcp_ftz((float)c.t));
    c.a1 = zero && c.t * s == T && c.t <= L;
    c.valid = c.a1 && xdiv && q * s == S && u * c.t == L;
    return c;
}

}  // namespace beast
