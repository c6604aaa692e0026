/*
 * beast.h — C ABI of the B200-native BEAST GEMM search-space enumerator.
 *
 * The library enumerates the 15-dimensional GEMM tuning space of Luszczek,
 * Gates, Kurzak, Danalis, Dongarra, "Search Space Generation and Pruning
 * System for Autotuners", IPDPSW 2016, applies its 12 pruning
 * predicates and returns the survivor count and the canonically ordered list
 * of surviving kernel variants.  Citations "P:<line>" are lines of PAPER.md.
 *
 *   space    Fig 8 device query, Fig 9 compute-capability lookups
 *            (P:932-957), Fig 10 settings, Fig 11 iterators
 *            (P:1041-1118), Fig 12 derived variables, Fig 14
 *            thresholds.
 *   pruning  Fig 13 hard, Fig 14 soft and Fig 15 correctness constraints
 *            (P:1265-1394); a constraint that evaluates True prunes the point
 *            (P:1243-1259, 1331-1349, 1363-1412).
 *
 * Conventions (all entry points):
 *   - extern "C", no exceptions cross the ABI; every function returns a
 *     beast_status (0 = BEAST_OK, negative = error).  Output parameters are
 *     written only on BEAST_OK, except that beast_enumerate* write *written
 *     on BEAST_ERR_CAPACITY (the required count; buffer contents unspecified).
 *   - `stream` is a cudaStream_t passed as void* (NULL = the legacy default
 *     stream).  Calls are stream-ordered and return after synchronising that
 *     stream, so host outputs are valid on return.
 *   - A beast_space handle owns its device scratch (allocated on first use,
 *     grown on demand, kept until beast_space_destroy) through the allocator
 *     set with beast_space_set_allocator (default cudaMalloc / cudaFree).  A
 *     handle is not safe for concurrent calls from several host threads;
 *     separate handles are independent.  The passes of one handle share its
 *     scratch, so a pass enqueued on a stream other than the previous pass's
 *     first waits (cudaStreamWaitEvent) for the end of that pass;
 *     beast_space_destroy waits for the handle's last pass before releasing
 *     the scratch.  Device calls run on the CUDA device current at call
 *     time, which must not change over the handle's life.
 *   - rank / world select a shard: the contiguous canonical range of L4
 *     survivors (dim_m, dim_n, blk_m, blk_n) whose cumulative estimated
 *     enumeration work falls in [W*rank/world, W*(rank+1)/world), with every
 *     point below them (L5-L15).  Levels L1-L4 run on every rank; their
 *     statistics are reported by rank 0 only.  The global survivor list is the
 *     concatenation of the shards in rank order.  world = 1, rank = 0 is the
 *     whole space.  The library never communicates between ranks.
 *   - There is no CPU fallback: every call that enumerates needs a CUDA
 *     device of compute capability 10.0 (sm_100a) and fails with
 *     BEAST_ERR_CUDA otherwise.
 */
#ifndef BEAST_H_
#define BEAST_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BEAST_ABI_VERSION 2

typedef enum {
    BEAST_OK = 0,
    BEAST_ERR_INVALID_ARGUMENT = -1, /* NULL pointer, bad rank/world, bad value */
    BEAST_ERR_UNSUPPORTED = -2,      /* a value outside the packed-record or kernel range */
    BEAST_ERR_CAPACITY = -3,         /* caller's record buffer too small; *written = required */
    BEAST_ERR_WORKSPACE = -4,        /* device scratch could not be allocated */
    BEAST_ERR_CUDA = -5              /* a CUDA runtime error (no device, launch failure, ...) */
} beast_status;

/* Device limits: the twelve values of Fig 8 as returned by
 * cudaGetDeviceProperties, then the three Fig 9 lookups.  A Fig 9
 * field <= 0 is resolved from the compute-capability tables of Fig 9
 * (cc 1.0-3.5) extended with a cc 10.0 row (32 blocks, 64 warps,
 * 255 registers; reading A10).  max_threads_per_multi_processor
 * and max_warps_per_multi_processor are carried but unused by Figs 12-15. */
typedef struct {
    int32_t max_threads_per_block;
    int32_t max_threads_dim_x;
    int32_t max_threads_dim_y;
    int32_t max_shared_mem_per_block;
    int32_t warp_size;
    int32_t max_regs_per_block;
    int32_t max_threads_per_multi_processor;
    int32_t cuda_major;
    int32_t cuda_minor;
    int32_t max_registers_per_multi_processor;
    int32_t max_shmem_per_multi_processor;
    int32_t float_size;
    int32_t max_blocks_per_multi_processor;   /* Fig 9, <= 0: look up */
    int32_t max_warps_per_multi_processor;    /* Fig 9, <= 0: look up */
    int32_t max_registers_per_thread;         /* Fig 9, <= 0: look up */
} beast_device_limits;

/* Fig 10 precision x arithmetic: single/real, double/real,
 * single/complex, double/complex.  Selects the dim_vec set (Fig 11
 * P:1052-1068, reading A1: S {1,4}, D {1,2}, C {1,2}, Z {1}) and the x2
 * factors of Fig 12. */
typedef enum { BEAST_SGEMM = 0, BEAST_DGEMM = 1, BEAST_CGEMM = 2, BEAST_ZGEMM = 3 } beast_precision;

/* Fig 10 transposes and Fig 14 thresholds. */
typedef struct {
    int32_t trans_a;                          /* 0 or 1 */
    int32_t trans_b;                          /* 0 or 1 */
    int32_t min_threads_per_multi_processor;  /* paper: 256 */
    int32_t min_fmas_per_load;                /* paper: 2 */
} beast_settings;

/* Upper limits of the five independent Fig 11 ranges.  A value
 * <= 0 selects the paper's default: dim_m <= max_threads_dim_x, dim_n <=
 * max_threads_dim_y, blk_m <= max_threads_dim_x, blk_n <= max_threads_dim_y,
 * blk_k <= min(max_threads_dim_x, max_threads_dim_y) (reading A9).  The
 * ranges of dim_m_a, dim_n_a, dim_m_b, dim_n_b follow from the blk values
 * (P:1079-1113). */
typedef struct {
    int32_t dim_m_max, dim_n_max, blk_m_max, blk_n_max, blk_k_max;
} beast_bounds;

/* Per-level and per-predicate counters of one call (this shard).
 * visits[l]: loop-body executions of level l+1 in Fig 11 order (L1 dim_m ..
 * L15 shmem_banks) under the canonical hoisted nest (reading A6).
 * rejected[i]: points whose first failing predicate is i, in the paper's
 * listing order Fig 13 -> 14 -> 15:
 *   0 over_max_threads  1 over_max_regs_per_thread  2 over_max_regs_per_block
 *   3 over_max_shmem  4 low_occupancy_regs  5 low_occupancy_shmem  6 low_fmas
 *   7 partial_warps  8 cant_reshape_a1  9 cant_reshape_b1  10 cant_reshape_a2
 *   11 cant_reshape_b2
 * Levels L1..L6 and predicates 0..7 are charged to rank 0 only (every rank
 * recomputes them); summing the stats of all ranks gives the whole space.
 * points_evaluated = sum(visits).
 *
 * Evaluation evidence (SURVEY §8(d) honesty rule: the instrumented run shows
 * what the timed run evaluates).  The A-read (L8-L9) and B-read (L10-L11)
 * grids of a job are evaluated row by row -- a row holds the short-axis
 * coordinate fixed and runs the long one over 1..L -- by a packed scan that
 * forms 16 points per loop iteration.  formed[s] (s = 0: A grids, 1: B
 * grids) counts 16 per executed iteration of every live row, counted inside
 * the scan loop, so formed[0] = sum over rows of 16 * ceil(L / 16) >=
 * visits[8] (the excess is each row's padding to whole 16-point blocks) and
 * likewise formed[1] >= visits[10].  checked[s]: rows whose scan found a
 * candidate zero and were then checked exactly (>= the a1 / b1 passes).
 * l4_digest: order-sensitive digest sum_i sm64(w_i ^ sm64(i)) of this call's
 * list of L4 survivors (levels L1-L4, computed redundantly by every rank:
 * equal on every rank of one space; sm64 as in beast_digest). */
typedef struct {
    uint64_t visits[15];
    uint64_t rejected[12];
    uint64_t survivors;
    uint64_t prefixes;          /* L7 prefixes in this shard */
    uint64_t valid_a;           /* (prefix, dim_m_a, dim_n_a) passing a1 and a2 */
    uint64_t tuples;            /* (prefix, A grid, B grid) survivors; survivors = 16 * tuples */
    uint64_t formed[2];         /* points formed by the packed scan, A / B grids (stats runs only) */
    uint64_t checked[2];        /* rows checked exactly, A / B grids (stats runs only) */
    uint64_t l4_digest;         /* digest of the L4 survivor list (every run) */
} beast_stats;

/* One surviving variant, 16 bytes, 16-byte aligned; as a little-endian
 * unsigned 128-bit integer (hi:lo) the canonical order (lexicographic over the
 * 15-tuple in Fig 11 order, all ranges ascending; reading A7) is ascending
 * numeric order.  Values are stored as-is (not minus one):
 *   hi[63:52] dim_m  hi[51:40] dim_n  hi[39:28] blk_m  hi[27:16] blk_n
 *   hi[15:4] blk_k   hi[3:1] dim_vec  hi[0] vec_mul
 *   lo[63:52] dim_m_a  lo[51:40] dim_n_a  lo[39:28] dim_m_b  lo[27:16] dim_n_b
 *   lo[15:4] 0  lo[3] tex_a  lo[2] tex_b  lo[1] shmem_l1  lo[0] shmem_banks */
typedef struct {
    uint64_t lo;
    uint64_t hi;
} beast_record;

typedef struct beast_space beast_space;   /* opaque, library-owned */

/* Device scratch allocator: alloc returns device memory of >= bytes usable on
 * `stream` (NULL on failure); free releases it.  ctx is passed through. */
typedef void *(*beast_alloc_fn)(size_t bytes, void *stream, void *ctx);
typedef void (*beast_free_fn)(void *ptr, size_t bytes, void *stream, void *ctx);

/* Library / ABI version (BEAST_ABI_VERSION). */
int beast_abi_version(void);

/* Human-readable text of a status code (static storage). */
const char *beast_error_string(int status);

/* Text of the last error recorded on this handle (empty if none). */
const char *beast_last_error(const beast_space *space);

/* Fig 8 values of a Tesla K40c with the Fig 9 fields resolved for
 * cc 3.5 (16 blocks, 64 warps, 255 registers).  out: caller-owned. */
int beast_limits_k40c(beast_device_limits *out);

/* Fig 8 values of CUDA device `device` from cudaGetDeviceProperties (
 * max_shared_mem_per_block = sharedMemPerBlockOptin, reading A10), Fig 9
 * fields from the table (or the device's maxBlocksPerMultiProcessor where the
 * table has no row).  BEAST_ERR_CUDA if the device cannot be queried. */
int beast_limits_from_device(int device, beast_device_limits *out);

/* Fill the Fig 9 fields of *limits that are <= 0 from the tables.
 * BEAST_ERR_UNSUPPORTED if the compute capability has no table row. */
int beast_limits_resolve(beast_device_limits *limits);

/* Create a space description.  settings / bounds may be NULL (trans 0/0,
 * thresholds 256/2; default bounds).  Validates and resolves the inputs on
 * the host only; no device work.  BEAST_ERR_UNSUPPORTED if a bound exceeds
 * 4095 (the 12-bit record fields), if max_threads_per_block > 65535,
 * max_blocks_per_multi_processor > 65534, float_size > 1024,
 * min_threads_per_multi_processor > 2^30 or min_fmas_per_load > 2^20 (the
 * ranges the packed words and the integer predicate arithmetic cover), or if
 * a limit is non-positive where the paper divides by it; BEAST_ERR_INVALID_ARGUMENT
 * for NULL limits/out or a bad precision.  *out: owned by the caller, release
 * with beast_space_destroy. */
int beast_space_create(const beast_device_limits *limits, beast_precision precision,
                       const beast_settings *settings, const beast_bounds *bounds,
                       beast_space **out);

/* Release a handle and its device scratch (NULL is ignored). */
void beast_space_destroy(beast_space *space);

/* Replace the scratch allocator (before the first enumerating call only;
 * BEAST_ERR_INVALID_ARGUMENT afterwards).  NULL fns restore cudaMalloc/Free. */
int beast_space_set_allocator(beast_space *space, beast_alloc_fn alloc, beast_free_fn free_fn,
                              void *ctx);

/* The resolved description actually enumerated (Fig 9 fields and default
 * bounds filled in).  Any out pointer may be NULL. */
int beast_space_resolved(const beast_space *space, beast_device_limits *limits,
                         beast_settings *settings, beast_bounds *bounds);

/* Count the survivors of shard (rank, world).  *survivors: host, out.
 * stats: host, out, nullable; non-NULL selects the instrumented kernels,
 * which execute the same evaluation and additionally count every loop-body
 * execution and first-failing predicate. */
int beast_count(beast_space *space, int rank, int world, void *stream,
                uint64_t *survivors, beast_stats *stats);

/* Enumerate the survivors of shard (rank, world) into `out`, a caller-owned
 * DEVICE buffer of `capacity` records, in canonical order.  *written: host,
 * out (records of this shard).  stats: as beast_count.
 * BEAST_ERR_CAPACITY if capacity < the shard's survivors. */
int beast_enumerate(beast_space *space, int rank, int world, void *stream,
                    beast_record *out, uint64_t capacity, uint64_t *written,
                    beast_stats *stats);

/* As beast_enumerate, but `host_out` is HOST memory (pinned for full copy
 * bandwidth); the list is produced in device scratch and copied back on
 * `stream`. */
int beast_enumerate_to_host(beast_space *space, int rank, int world, void *stream,
                            beast_record *host_out, uint64_t capacity, uint64_t *written,
                            beast_stats *stats);

/* Stream-ordered enumeration without a host wait.  Enqueues on `stream` the
 * pass that an earlier synchronous beast_enumerate captured for the same
 * (rank, world, out, capacity) -- stats off, the handle's current timing
 * setting -- and returns at once; `out` is complete when the stream reaches
 * the end of the pass.  Passes on one handle must be issued from one host
 * thread.  BEAST_ERR_INVALID_ARGUMENT if no such captured pass exists (call
 * beast_enumerate first). */
int beast_enumerate_async(beast_space *space, int rank, int world, void *stream,
                          beast_record *out, uint64_t capacity);

/* Host-buffer enumeration without a host wait, for pipelining passes of
 * several handles against their device -> host copies (the copy engine moves
 * one list over PCIe while the SMs compute the next).  Enqueues on `stream`
 * the pass that the last successful beast_enumerate_to_host of this handle
 * captured for (rank, world) -- same device staging buffer, stats off --
 * followed by the copy of its records into `host_out` (HOST memory of
 * `capacity` records; pinned, or the copy is not asynchronous), and returns
 * at once.  The copy length is that earlier call's record count: a handle's
 * space is fixed, so every pass of one (rank, world) yields the same list;
 * beast_wait checks it.  `host_out` is valid after beast_wait returns
 * BEAST_OK.  Errors: BEAST_ERR_INVALID_ARGUMENT if there was no such earlier
 * call, BEAST_ERR_CAPACITY if its count exceeds `capacity` (nothing is
 * enqueued). */
int beast_enumerate_to_host_async(beast_space *space, int rank, int world, void *stream,
                                  beast_record *host_out, uint64_t capacity);

/* Wait for the most recent pass of the handle (synchronous or asynchronous)
 * to complete -- and, after beast_enumerate_to_host_async, its host copy;
 * *written: host, out, the records of that pass.  BEAST_ERR_CAPACITY if they
 * exceeded the capacity of that pass's record buffer (counting passes have
 * none); BEAST_ERR_WORKSPACE if
 * an asynchronous pass overflowed its scratch or a host pass's count differed
 * from the copied one. */
int beast_wait(beast_space *space, void *stream, uint64_t *written);

/* fused survivor gather (the writer
 * stores the shard's records straight into rank 0's buffer at the shard's
 * global offset, over NVLink, instead of a separate NCCL gather).
 *
 * beast_enumerate_stage: run shard (rank, world)'s pass up to its canonical
 * tuple list (prefix stage, flattener, A and B grids, canonical placement;
 * no write-out) and store the shard's record count (16 per tuple) into
 * *d_count, a caller-owned DEVICE u64 (8-byte aligned), on `stream`.
 * *count: host, out, nullable (the same number).  Synchronous.
 *
 * beast_write_at: write-out of the staged shard (the last pass on this
 * handle must be beast_enumerate_stage with the same rank, world): record i
 * of the shard is stored at out[base + i], base = d_counts[0] + ... +
 * d_counts[rank - 1], where d_counts is a DEVICE array of `world` u64
 * (typically the all-gather of every rank's *d_count, produced on `stream`).
 * `out` is a DEVICE pointer valid in this process -- rank 0's output buffer
 * mapped into it (CUDA IPC / symmetric memory over NVLink) or a local buffer;
 * `capacity` = records it holds (16-byte aligned).  *base_out: host, out,
 * nullable.  Reads d_counts back (one small stream-synchronous copy), then
 * enqueues the write-out kernel and returns; the records are complete when
 * `stream` reaches it.  The concatenation over ranks equals the world-1
 * list.  Errors: BEAST_ERR_INVALID_ARGUMENT (nothing staged for (rank,
 * world), d_counts[rank] differs from the staged count), BEAST_ERR_CAPACITY
 * (base + count > capacity; nothing written). */
int beast_enumerate_stage(beast_space *space, int rank, int world, void *stream, uint64_t *d_count,
                          uint64_t *count);
int beast_write_at(beast_space *space, int rank, int world, void *stream, beast_record *out,
                   uint64_t capacity, const uint64_t *d_counts, uint64_t *base_out);

/* batched sweep: count the survivors of n independent
 * spaces in one call, e.g. the 4 precisions x 4 transposes x {K40c, B200}
 * configurations the paper tunes one at a time (Fig 10).
 * Each space's counting pass (the same kernels as beast_count, rank 0 of
 * world 1) is launched on one of a pool of internal streams forked from
 * `stream` and joined back to it, so the spaces' passes run concurrently;
 * then every handle's counters are read.  spaces: host array of n distinct
 * handles on the current device.  survivors: host, out, n entries.
 * stats: host, out, n entries or NULL; non-NULL selects the instrumented
 * passes, and each entry is then the space's per-level visits and
 * first-failing-predicate rejections (Figs 11-15) -- the attribution table
 * of the sweep.  A handle without a captured counting pass first runs one
 * synchronous beast_count.  Errors: BEAST_ERR_INVALID_ARGUMENT (NULL or
 * repeated handle, handle on another device), any beast_count error. */
int beast_sweep_count(beast_space *const *spaces, int n, void *stream, uint64_t *survivors,
                      beast_stats *stats);

/* generic space IR.  A space written the way the
 * BEAST language writes one (§V-VIII): iterators whose
 * [start, stop) ranges with a step are C int64 expressions of constants and
 * earlier iterators (values start, start+step, ... while < stop for step > 0,
 * > stop for step < 0), derived variables (C int64 expressions, listing
 * order) and constraints (C expressions; nonzero prunes, reading A5).  Every
 * derived variable and constraint belongs to the deepest iterator it reads
 * (the level-set rule); constraints of one level are tested in
 * listing order and the first that holds is the point's rejection.  All
 * strings are copied; names are C identifiers; an expression may read only
 * names declared before it (in the level sense).  Arithmetic is C int64 (/
 * and % truncate; an expression must not divide by zero -- guard it with
 * || or ?:, e.g. "loads == 0 || fmas / loads < 2"). */
typedef struct beast_ir beast_ir;   /* opaque, library-owned */
typedef struct {
    int32_t n_constants;
    const char *const *constant_names;
    const int64_t *constant_values;
    int32_t n_iterators;                          /* <= 64 */
    const char *const *iterator_names;
    const char *const *iterator_start, *const *iterator_stop, *const *iterator_step;
    int32_t n_derived;
    const char *const *derived_names;
    const char *const *derived_exprs;
    int32_t n_constraints;                        /* <= 64 */
    const char *const *constraint_names;
    const char *const *constraint_exprs;
} beast_ir_desc;

/* Validate, assign levels, generate the CUDA source of the space and compile
 * it for sm_100a with NVRTC (opened at run time; BEAST_NVRTC may name the
 * library).  Needs no GPU: the cubin is loaded on the current device by the
 * first count / enumerate.  On failure *out may still receive a
 * handle whose beast_ir_last_error explains it (destroy it).  Errors:
 * BEAST_ERR_INVALID_ARGUMENT (bad name, unknown or later-level name in an
 * expression, NVRTC compile error), BEAST_ERR_UNSUPPORTED (no NVRTC),
 * BEAST_ERR_CUDA. */
int beast_ir_create(const beast_ir_desc *desc, beast_ir **out);
void beast_ir_destroy(beast_ir *ir);
const char *beast_ir_last_error(const beast_ir *ir);
/* The generated CUDA source (owned by the handle). */
const char *beast_ir_source(const beast_ir *ir);
/* Level (0-based iterator index, -1 = constants only) of every derived
 * variable and constraint; host arrays, nullable. */
int beast_ir_levels(const beast_ir *ir, int32_t *derived_levels, int32_t *constraint_levels);
/* Count the survivors level by level on `stream` (synchronous).  visits: host,
 * out, n_iterators loop-body executions per level, nullable; rejected: host,
 * out, n_constraints first-failing counts, nullable. */
int beast_ir_count(beast_ir *ir, void *stream, uint64_t *survivors, uint64_t *visits, uint64_t *rejected);
/* As beast_ir_count, and write the survivors in canonical (lexicographic,
 * listing-order) order into `out`, a DEVICE buffer of `capacity` rows of
 * n_iterators int64 values.  *written = survivors.  BEAST_ERR_CAPACITY if
 * capacity < survivors (nothing of the last level written).  Intermediate
 * levels are materialised in stream-ordered device allocations
 * (BEAST_ERR_WORKSPACE if one does not fit). */
int beast_ir_enumerate(beast_ir *ir, void *stream, int64_t *out, uint64_t capacity, uint64_t *written,
                       uint64_t *visits, uint64_t *rejected);

/* factorised evaluation (time to solution; NOT the
 * canonical points/s path): the A and B read-grid sub-nests of a prefix are
 * independent level sets (§X-B) and cant_reshape_a1/b1
 * can only be False where dim_m_x * dim_n_x == threads_per_block,
 * so each prefix's valid A and B grids are found among the divisors of T and
 * its survivors are their product.  Same survivor count / canonical list as
 * beast_count / beast_enumerate (checked by the parity tests); no per-point
 * evaluation and therefore no stats.  Arguments as beast_count /
 * beast_enumerate. */
int beast_count_factorized(beast_space *space, int rank, int world, void *stream, uint64_t *survivors);
int beast_enumerate_factorized(beast_space *space, int rank, int world, void *stream, beast_record *out,
                               uint64_t capacity, uint64_t *written);

/* Order-sensitive digest of n device records:
 *   sum_i sm64(sm64(hi_i ^ sm64(base + i)) ^ lo_i) mod 2^64,
 * sm64 = splitmix64 finaliser.  Partial digests of consecutive shards (with
 * base = the shard's global offset) add up to the digest of the whole list.
 * records: device, read only.  *digest: host, out. */
int beast_digest(const beast_record *records, uint64_t n, uint64_t base, void *stream,
                 uint64_t *digest);

/* Device time in milliseconds of the stages of the last call on this handle
 * (CUDA events): [0] prefix stage L1-L7, [1] flattener + A grids L8-L9,
 * [2] B grids L10-L11, [3] compaction + write-out, [4] whole call.
 * Timing events are recorded only when enabled (beast_space_set_timing). */
int beast_space_set_timing(beast_space *space, int enable);
int beast_last_stage_ms(const beast_space *space, float ms[5]);

/* Launch statistics of the last call: number of kernels launched and the
 * average duration (ms, CUDA events on the launching stream, timing enabled
 * only) of the dominant kernel (the A-grid evaluation). */
int beast_last_launches(const beast_space *space, uint64_t *kernels, float *a_eval_ms,
                        uint64_t *a_eval_launches);

/* Device time in milliseconds (CUDA events on the launching stream, timing
 * enabled) of the survivor write-out kernel (§8(a) a7: 16 packed 16-byte
 * records per surviving tuple) of the last synchronous beast_enumerate /
 * beast_enumerate_to_host on this handle; -1 if that call wrote no list or
 * timing was off.  *ms: host, out. */
int beast_last_write_ms(const beast_space *space, float *ms);

/* beast_stats.l4_digest of the last completed pass on this handle (any mode,
 * stats or not): the digest of its L4 survivor list, which every rank of a
 * sharded run computes redundantly -- the multi-GPU combine all-gathers it
 * and checks that the ranks agree.  *digest: host, out.
 * BEAST_ERR_INVALID_ARGUMENT before the first pass. */
int beast_last_l4_digest(const beast_space *space, uint64_t *digest);

#ifdef __cplusplus
}
#endif

#endif /* BEAST_H_ */
