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

__device__ __forceinline__ uint64_t ld_volatile_u64(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ void st_volatile_u64(uint64_t *p, uint64_t v) {
    asm volatile("st.volatile.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// --------------------------------------------- decoupled look-back prefix
// Tile status word: [63:62] flag (0 empty, 1 aggregate, 2 inclusive prefix),
// [61:0] value.  Tiles are handed out in increasing order by an atomic
// counter, so every predecessor of a tile is owned by a resident CTA and the
// look-back always terminates.
constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagInc = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;

// Called by ALL 32 lanes of one warp.  Publishes `aggregate` for `tile` and
// returns the exclusive prefix of all earlier tiles.
__device__ __forceinline__ uint64_t lookback_exclusive(uint64_t *status, uint64_t tile,
                                                       uint64_t aggregate) {
    const uint32_t lane = lane_id();
    if (tile == 0) {
        if (lane == 0) st_volatile_u64(&status[0], kFlagInc | aggregate);
        return 0;
    }
    if (lane == 0) st_volatile_u64(&status[tile], kFlagAgg | aggregate);
    uint64_t exclusive = 0;
    int64_t base = (int64_t)tile - 1;
    while (true) {
        const int64_t t = base - (int64_t)lane;
        uint64_t s = t >= 0 ? ld_volatile_u64(&status[t]) : kFlagInc;
        while (__any_sync(kFull, (s >> 62) == 0)) {
            if ((s >> 62) == 0) s = ld_volatile_u64(&status[t]);
        }
        const uint32_t inc = __ballot_sync(kFull, (s >> 62) == 2);
        const int stop = inc ? __ffs(inc) - 1 : 32;
        const uint64_t v = (int)lane <= stop ? (s & kValMask) : 0;
        exclusive += warp_sum_u64(v);
        if (inc) break;
        base -= 32;
    }
    if (lane == 0) st_volatile_u64(&status[tile], kFlagInc | (exclusive + aggregate));
    return exclusive;
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
// Evaluates cant_reshape_{a,b}1, "dim_m_x * dim_n_x !=
// threads_per_block", on 16 consecutive points of one grid row: the row
// holds the short-axis coordinate `s` fixed and runs the long-axis
// coordinate over base/s + 1 .. base/s + 16, so the products are
// base + s*1 .. base + s*16.  One IMAD (FMA pipe) forms each product and one
// ISETP.EQ.OR (ALU pipe) compares it with T and folds it into the row's hit
// predicate: two issue slots per point, the two pipes evenly loaded.
__device__ __forceinline__ uint32_t eval16(uint32_t hit, uint32_t base, uint32_t s, uint32_t T) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .u32 t<16>;\n\t"
        "setp.ne.u32 p, %0, 0;\n\t"
        "mad.lo.u32 t0, %2, 1, %1;\n\t setp.eq.or.u32 p, t0, %3, p;\n\t"
        "mad.lo.u32 t1, %2, 2, %1;\n\t setp.eq.or.u32 p, t1, %3, p;\n\t"
        "mad.lo.u32 t2, %2, 3, %1;\n\t setp.eq.or.u32 p, t2, %3, p;\n\t"
        "mad.lo.u32 t3, %2, 4, %1;\n\t setp.eq.or.u32 p, t3, %3, p;\n\t"
        "mad.lo.u32 t4, %2, 5, %1;\n\t setp.eq.or.u32 p, t4, %3, p;\n\t"
        "mad.lo.u32 t5, %2, 6, %1;\n\t setp.eq.or.u32 p, t5, %3, p;\n\t"
        "mad.lo.u32 t6, %2, 7, %1;\n\t setp.eq.or.u32 p, t6, %3, p;\n\t"
        "mad.lo.u32 t7, %2, 8, %1;\n\t setp.eq.or.u32 p, t7, %3, p;\n\t"
        "mad.lo.u32 t8, %2, 9, %1;\n\t setp.eq.or.u32 p, t8, %3, p;\n\t"
        "mad.lo.u32 t9, %2, 10, %1;\n\t setp.eq.or.u32 p, t9, %3, p;\n\t"
        "mad.lo.u32 t10, %2, 11, %1;\n\t setp.eq.or.u32 p, t10, %3, p;\n\t"
        "mad.lo.u32 t11, %2, 12, %1;\n\t setp.eq.or.u32 p, t11, %3, p;\n\t"
        "mad.lo.u32 t12, %2, 13, %1;\n\t setp.eq.or.u32 p, t12, %3, p;\n\t"
        "mad.lo.u32 t13, %2, 14, %1;\n\t setp.eq.or.u32 p, t13, %3, p;\n\t"
        "mad.lo.u32 t14, %2, 15, %1;\n\t setp.eq.or.u32 p, t14, %3, p;\n\t"
        "mad.lo.u32 t15, %2, 16, %1;\n\t setp.eq.or.u32 p, t15, %3, p;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "+r"(hit)
        : "r"(base), "r"(s), "r"(T));
    return hit;
}

// Whole row of L points: products s*1 .. s*L compared with T.
__device__ __forceinline__ uint32_t eval_row(uint32_t s, uint32_t T, uint32_t L) {
    uint32_t hit = 0, base = 0, j = 0;
    for (; j + 16 <= L; j += 16) {
        hit = eval16(hit, base, s, T);
        base += 16u * s;
    }
    for (; j < L; ++j) {
        base += s;
        hit |= (base == T);
    }
    return hit;
}

}  // namespace beast
