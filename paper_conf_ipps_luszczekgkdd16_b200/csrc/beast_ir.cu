// beast_ir.cu — SURVEY §8(f) NEXT #4: the generic space IR.
//
// A space is written the way the BEAST language writes one (§V-VIII,
// P:365-770): iterators whose ranges are expressions of earlier iterators,
// derived variables (expressions) and constraints (True prunes, reading A5).
// beast_ir_create checks the description, assigns every derived variable and
// constraint to the deepest iterator it reads (the level-set rule of §X-B,
// P:1576-1594), generates one CUDA translation unit -- the range and
// constraint functions of every level followed by a fixed level-wise
// enumeration engine -- and compiles it for sm_100a with NVRTC at run time
// (libnvrtc is opened with dlopen, so the library still loads on a machine
// without a GPU).  The engine enumerates level by level in canonical
// (lexicographic) order: per level, one warp per parent tuple counts the
// values of the level's iterator that pass the level's constraints (first
// failing constraint attributed, listing order), an exclusive scan gives
// offsets, and one warp per parent re-evaluates and writes the child tuples
// at offset + warp rank -- the nested-emission scheme of the GEMM prefix
// stage (beast_kernels.cuh), generic over the compiled functions.
//
// This file shares nothing with oracle/ir.py (which writes the same
// description out as plain C nested loops for gcc).

#include "beast.h"

#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <set>
#include <string>
#include <vector>

namespace {

// ------------------------------------------------------------ NVRTC (dlopen)
typedef int nvrtcResult_t;
typedef struct _nvrtcProgram *nvrtcProgram_t;
struct Nvrtc {
    bool ok = false;
    nvrtcResult_t (*create)(nvrtcProgram_t *, const char *, const char *, int, const char *const *,
                            const char *const *) = nullptr;
    nvrtcResult_t (*compile)(nvrtcProgram_t, int, const char *const *) = nullptr;
    nvrtcResult_t (*log_size)(nvrtcProgram_t, size_t *) = nullptr;
    nvrtcResult_t (*log)(nvrtcProgram_t, char *) = nullptr;
    nvrtcResult_t (*cubin_size)(nvrtcProgram_t, size_t *) = nullptr;
    nvrtcResult_t (*cubin)(nvrtcProgram_t, char *) = nullptr;
    nvrtcResult_t (*destroy)(nvrtcProgram_t *) = nullptr;
    const char *(*errstr)(nvrtcResult_t) = nullptr;
};

Nvrtc &nvrtc() {
    static Nvrtc n;
    static std::once_flag once;
    std::call_once(once, [] {
        const char *env = getenv("BEAST_NVRTC");
        const char *cands[] = {env, "libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so",
                               "/usr/local/cuda/lib64/libnvrtc.so"};
        void *h = nullptr;
        for (const char *c : cands)
            if (c && (h = dlopen(c, RTLD_NOW | RTLD_LOCAL))) break;
        if (!h) return;
        auto sym = [&](const char *s) { return dlsym(h, s); };
        n.create = (decltype(n.create))sym("nvrtcCreateProgram");
        n.compile = (decltype(n.compile))sym("nvrtcCompileProgram");
        n.log_size = (decltype(n.log_size))sym("nvrtcGetProgramLogSize");
        n.log = (decltype(n.log))sym("nvrtcGetProgramLog");
        n.cubin_size = (decltype(n.cubin_size))sym("nvrtcGetCUBINSize");
        n.cubin = (decltype(n.cubin))sym("nvrtcGetCUBIN");
        n.destroy = (decltype(n.destroy))sym("nvrtcDestroyProgram");
        n.errstr = (decltype(n.errstr))sym("nvrtcGetErrorString");
        n.ok = n.create && n.compile && n.log_size && n.log && n.cubin_size && n.cubin && n.destroy;
    });
    return n;
}

// ------------------------------------------------------------ the engine
// Fixed helpers placed before the generated per-level kernels (see
// generate()): trip count of a range, warp sum, the three-phase scan.
const char *kEngine = R"CUDA(
typedef unsigned long long u64;

__device__ __forceinline__ u64 ir_trip(i64 lo, i64 hi, i64 st) {
    if (st > 0) return hi > lo ? (u64)((hi - lo + st - 1) / st) : 0ull;
    return lo > hi ? (u64)((lo - hi - st - 1) / (-st)) : 0ull;
}

__device__ __forceinline__ u64 warp_sum(u64 x) {
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}

// Exclusive scan of n counts, three phases (tiles of 2048 = 256 x 8).
extern "C" __global__ void __launch_bounds__(256) ir_scan_tiles(const u64 *in, u64 n, u64 *out, u64 *tile_sum) {
    __shared__ u64 s_w[8];
    const u64 t0 = (u64)blockIdx.x * 2048 + threadIdx.x * 8;
    u64 x[8], s = 0;
    for (int i = 0; i < 8; ++i) { x[i] = t0 + i < n ? in[t0 + i] : 0ull; s += x[i]; }
    const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    u64 inc = s;
    for (int o = 1; o < 32; o <<= 1) { const u64 y = __shfl_up_sync(0xffffffffu, inc, o); if ((int)lane >= o) inc += y; }
    if (lane == 31) s_w[warp] = inc;
    __syncthreads();
    u64 wb = 0;
    for (int w = 0; w < (int)warp; ++w) wb += s_w[w];
    u64 run = wb + inc - s;
    for (int i = 0; i < 8; ++i) { if (t0 + i < n) out[t0 + i] = run; run += x[i]; }
    if (threadIdx.x == 255) tile_sum[blockIdx.x] = wb + inc;
}
extern "C" __global__ void __launch_bounds__(1024) ir_scan_top(u64 *tile_sum, u64 n_tiles, u64 *total) {
    __shared__ u64 s_w[32];
    __shared__ u64 s_carry;
    const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) s_carry = 0;
    __syncthreads();
    for (u64 b = 0; b < n_tiles; b += 1024) {
        const u64 i = b + threadIdx.x;
        const u64 x = i < n_tiles ? tile_sum[i] : 0ull;
        u64 inc = x;
        for (int o = 1; o < 32; o <<= 1) { const u64 y = __shfl_up_sync(0xffffffffu, inc, o); if ((int)lane >= o) inc += y; }
        if (lane == 31) s_w[warp] = inc;
        __syncthreads();
        if (warp == 0) {
            u64 w = s_w[lane];
            for (int o = 1; o < 32; o <<= 1) { const u64 y = __shfl_up_sync(0xffffffffu, w, o); if ((int)lane >= o) w += y; }
            s_w[lane] = w;
        }
        __syncthreads();
        const u64 carry = s_carry;
        if (i < n_tiles) tile_sum[i] = carry + (warp ? s_w[warp - 1] : 0ull) + inc - x;
        __syncthreads();
        if (threadIdx.x == 0) s_carry = carry + s_w[31];
        __syncthreads();
    }
    if (threadIdx.x == 0) *total = s_carry;
}
extern "C" __global__ void __launch_bounds__(256) ir_scan_add(u64 *out, u64 n, const u64 *tile_sum, const u64 *total) {
    const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) out[i] += tile_sum[i / 2048];
    if (i == 0) out[n] = *total;
}
)CUDA";

bool is_ident_start(char c) { return (c >= 'a' && c <= 'z') || (c >= 'A' && c <= 'Z') || c == '_'; }
bool is_ident_char(char c) { return is_ident_start(c) || (c >= '0' && c <= '9'); }

std::vector<std::string> idents(const std::string &e) {
    std::vector<std::string> out;
    for (size_t i = 0; i < e.size();) {
        if (is_ident_start(e[i]) && (i == 0 || !is_ident_char(e[i - 1]))) {
            size_t j = i;
            while (j < e.size() && is_ident_char(e[j])) ++j;
            out.push_back(e.substr(i, j - i));
            i = j;
        } else {
            ++i;
        }
    }
    return out;
}

bool valid_name(const char *s) {
    if (!s || !is_ident_start(s[0])) return false;
    // the generated code's own names start with "ir_"; i64 / u64 are its types
    if (!strncmp(s, "ir_", 3) || !strcmp(s, "i64") || !strcmp(s, "u64")) return false;
    for (const char *p = s; *p; ++p)
        if (!is_ident_char(*p)) return false;
    return strlen(s) < 64;
}

}  // namespace

struct beast_ir {
    int ni = 0, nc = 0;
    std::vector<std::string> cnames, inames, dnames, knames;
    std::vector<long long> cvals;
    std::vector<std::string> istart, istop, istep, dexpr, kexpr;
    std::vector<int> dlev, klev;
    std::string src;
    std::vector<char> cubin;    // NVRTC output; loaded on the first run (create needs no GPU)
    std::string err;
    int device = -1;
    cudaLibrary_t lib = nullptr;
    std::vector<cudaKernel_t> k_count, k_emit;     // per level, warp per parent
    std::vector<cudaKernel_t> k_tcount, k_temit;   // per level, thread per parent
    std::vector<cudaKernel_t> k_fcount, k_femit;   // levels k and k + 1 fused (k without constraints), else null
    std::vector<cudaKernel_t> k_wfcount, k_wfemit; // the same, warp per parent
    cudaKernel_t k_root = nullptr, k_tiles = nullptr, k_top = nullptr,
                 k_add = nullptr;
    // kernel-shape choices learnt from the previous run of this handle:
    // average trip count of each level's iterator (values evaluated per
    // parent; < 0: unknown) and the fuse decision of each fusable level
    // (-1 unknown, 0 / 1)
    std::vector<double> avg_trip;
    std::vector<int> fuse_known;
    // the previous run's level totals (children surviving through level k,
    // ~0: not seen), its root pruning and static trip counts: a space is
    // fixed, so a later run enqueues every level without waiting for the
    // host (one synchronisation at the end, which checks these totals)
    std::vector<unsigned long long> known_tot, known_trip;
    int known_pruned = -1;
    int sm_count = 148;
};

namespace {

#define IRCK(x)                                                                                     \
    do {                                                                                            \
        cudaError_t e_ = (x);                                                                       \
        if (e_ != cudaSuccess) {                                                                    \
            ir->err = std::string(#x) + ": " + cudaGetErrorString(e_);                              \
            return BEAST_ERR_CUDA;                                                                  \
        }                                                                                           \
    } while (0)

// Level of each derived variable / constraint; validation of every name.
int analyse(beast_ir *ir) {
    std::map<std::string, int> lev;   // -1 = constant level
    std::set<std::string> seen;
    auto add = [&](const std::string &n, int l) -> bool {
        if (!seen.insert(n).second) {
            ir->err = "duplicate name " + n;
            return false;
        }
        lev[n] = l;
        return true;
    };
    auto level_of = [&](const std::string &e, int limit, const char *what) -> int {
        int l = -1;
        for (const auto &id : idents(e)) {
            auto it = lev.find(id);
            if (it == lev.end()) {
                ir->err = std::string("unknown name '") + id + "' in " + what + " expression '" + e + "'";
                return -2;
            }
            l = std::max(l, it->second);
        }
        if (l >= limit) {
            ir->err = std::string("expression '") + e + "' of " + what + " reads a variable of its own or a later level";
            return -2;
        }
        return l;
    };
    for (size_t i = 0; i < ir->cnames.size(); ++i)
        if (!add(ir->cnames[i], -1)) return BEAST_ERR_INVALID_ARGUMENT;
    // Declaration before use: a derived variable reads constants, iterators
    // and derived variables listed before it; its level is the deepest
    // iterator it reads (directly or through them).  An iterator's range reads
    // only names of earlier levels.
    std::map<std::string, int> iter_index;
    for (int k = 0; k < ir->ni; ++k) iter_index[ir->inames[k]] = k;
    std::vector<int> dl(ir->dnames.size(), -1);
    for (size_t d = 0; d < ir->dnames.size(); ++d) {
        int l = -1;
        for (const auto &id : idents(ir->dexpr[d])) {
            auto it = lev.find(id);
            int li;
            if (it != lev.end()) li = it->second;
            else if (iter_index.count(id)) li = iter_index[id];
            else {
                ir->err = "unknown (or not yet declared) name '" + id + "' in derived variable " + ir->dnames[d];
                return BEAST_ERR_INVALID_ARGUMENT;
            }
            l = std::max(l, li);
        }
        dl[d] = l;
        if (!add(ir->dnames[d], l)) return BEAST_ERR_INVALID_ARGUMENT;
    }
    for (int k = 0; k < ir->ni; ++k) {
        if (!add(ir->inames[k], k)) return BEAST_ERR_INVALID_ARGUMENT;
    }
    for (int k = 0; k < ir->ni; ++k)
        for (const std::string *e : {&ir->istart[k], &ir->istop[k], &ir->istep[k]})
            if (level_of(*e, k, "iterator range") == -2) return BEAST_ERR_INVALID_ARGUMENT;
    ir->dlev = dl;
    ir->klev.resize(ir->kexpr.size());
    for (size_t c = 0; c < ir->kexpr.size(); ++c) {
        const int l = level_of(ir->kexpr[c], 1 << 30, "constraint");
        if (l == -2) return BEAST_ERR_INVALID_ARGUMENT;
        ir->klev[c] = l;
        if (!valid_name(ir->knames[c].c_str())) {
            ir->err = "bad constraint name";
            return BEAST_ERR_INVALID_ARGUMENT;
        }
    }
    return BEAST_OK;
}

// Per level k the generated unit holds two kernels, specialised for the
// level (names bound as C locals, nothing indexed at run time):
//   ir_count_<k>: one warp per parent tuple (row of k values); binds the
//     parent's iterators and every derived variable of a shallower level ONCE
//     per parent, evaluates the range of iterator k, then lane-strided over
//     its values binds the level's derived variables and tests the level's
//     constraints in listing order (the first that holds is the rejection);
//     children per parent -> cnt, visits and rejections -> stats.
//   ir_emit_<k>: the same evaluation, writing the surviving child rows
//     (k + 1 values) at off[parent] + warp rank: canonical order.
// ir_root tests the constant-level constraints once.
std::string generate(const beast_ir *ir) {
    std::string s;
    char buf[512];
    s += "// generated by beast_ir_create (SURVEY §8(f) NEXT #4)\n";
    s += "typedef long long i64;\n";
    snprintf(buf, sizeof(buf), "#define NI %d\n#define NC %d\n", ir->ni, ir->nc);
    s += buf;
    s += kEngine;
    std::string consts;
    for (size_t i = 0; i < ir->cnames.size(); ++i) {
        snprintf(buf, sizeof(buf), "    const i64 %s = (i64)(%lldLL); (void)%s;\n", ir->cnames[i].c_str(),
                 ir->cvals[i], ir->cnames[i].c_str());
        consts += buf;
    }
    auto derived_at = [&](int lo, int hi, const char *ind) {   // derived variables with lo <= level <= hi
        std::string c;
        for (size_t d = 0; d < ir->dnames.size(); ++d)
            if (ir->dlev[d] >= lo && ir->dlev[d] <= hi)
                c += std::string(ind) + "const i64 " + ir->dnames[d] + " = (i64)(" + ir->dexpr[d] + "); (void)" +
                     ir->dnames[d] + ";\n";
        return c;
    };
    // first-failing counters of a level's nck constraints: registers (a
    // dynamically indexed array would live in local memory)
    auto rej_decl = [&](int nck) {
        std::string c = "";
        for (int l = 0; l < nck; ++l) c += "    u64 ir_rej" + std::to_string(l) + "_ = 0;\n";
        return c;
    };
    auto rej_inc = [&](int nck, const char *ind) {
        std::string c = std::string(ind) + "if (ir_r_ == 0) ++ir_c_;\n";
        for (int l = 0; l < nck; ++l)
            c += std::string(ind) + "else if (ir_r_ == " + std::to_string(l + 1) + ") ++ir_rej" + std::to_string(l) + "_;\n";
        return c;
    };
    auto constraints_at = [&](int k, const char *ind, std::vector<int> *idx) {
        std::string c;
        int local = 0;
        for (size_t j = 0; j < ir->kexpr.size(); ++j)
            if (ir->klev[j] == k) {
                ++local;
                c += std::string(ind) + (local == 1 ? "if" : "else if") + " ((" + ir->kexpr[j] + ")) ir_r_ = " +
                     std::to_string(local) + ";   // " + ir->knames[j] + "\n";
                if (idx) idx->push_back((int)j);
            }
        return c;
    };
    // root: constant-level constraints
    {
        std::vector<int> idx;
        s += "extern \"C\" __global__ void ir_root(u64 *ir_stats_, int *ir_pruned_, u64 *ir_trip_) {\n";
        s += consts + derived_at(-1, -1, "    ");
        // trip count of every iterator whose range depends on constants only
        // (the engine runs such short levels one thread per parent)
        for (int k = 0; k < ir->ni; ++k) {
            bool constant = true;
            for (const std::string *e : {&ir->istart[k], &ir->istop[k], &ir->istep[k]})
                for (const std::string &id : idents(*e)) {
                    bool ok = std::find(ir->cnames.begin(), ir->cnames.end(), id) != ir->cnames.end();
                    for (size_t d = 0; d < ir->dnames.size() && !ok; ++d)
                        ok = ir->dnames[d] == id && ir->dlev[d] < 0;
                    constant = constant && ok;
                }
            if (constant)
                s += "    { const i64 ir_st_ = (i64)(" + ir->istep[k] + "); ir_trip_[" + std::to_string(k) +
                     "] = ir_st_ == 0 ? 0ull : ir_trip((i64)(" + ir->istart[k] + "), (i64)(" + ir->istop[k] +
                     "), ir_st_); }\n";
            else
                s += "    ir_trip_[" + std::to_string(k) + "] = ~0ull;\n";
        }
        s += "    int ir_r_ = 0;\n" + constraints_at(-1, "    ", &idx);
        s += "    int ir_g_ = 0;\n";
        for (size_t l = 0; l < idx.size(); ++l)
            s += "    if (ir_r_ == " + std::to_string(l + 1) + ") ir_g_ = " + std::to_string(idx[l] + 1) + ";\n";
        s += "    *ir_pruned_ = ir_g_;\n    if (ir_g_) ir_stats_[NI + ir_g_ - 1] += 1;\n}\n";
    }
    for (int k = 0; k < ir->ni; ++k) {
        std::vector<int> idx;
        const std::string cons = constraints_at(k, "            ", &idx);
        const int nck = (int)idx.size();
        std::string parent;   // per-parent bindings
        for (int j = 0; j < k; ++j) {
            snprintf(buf, sizeof(buf), "        const i64 %s = ir_par_[ir_p_ * %d + %d]; (void)%s;\n",
                     ir->inames[j].c_str(), k, j, ir->inames[j].c_str());
            parent += buf;
        }
        parent += derived_at(-1, k - 1, "        ");
        parent += "        const i64 ir_lo_ = (i64)(" + ir->istart[k] + "), ir_hi_ = (i64)(" + ir->istop[k] +
                  "), ir_st_ = (i64)(" + ir->istep[k] + ");\n";
        parent += "        const u64 ir_n_ = ir_st_ == 0 ? 0ull : ir_trip(ir_lo_, ir_hi_, ir_st_);\n";
        std::string point;   // per-value bindings + constraints
        point += "            const i64 " + ir->inames[k] + " = ir_lo_ + (i64)ir_i_ * ir_st_; (void)" +
                 ir->inames[k] + ";\n";
        point += derived_at(k, k, "            ");
        point += "            int ir_r_ = 0;\n" + cons;
        const std::string head =
            "    const unsigned ir_lane_ = threadIdx.x & 31;\n"
            "    const u64 ir_w0_ = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;\n"
            "    const u64 ir_nw_ = ((u64)gridDim.x * blockDim.x) >> 5;\n";
        // count
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_count_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "u64 *ir_cnt_, u64 *ir_stats_) {\n", k);
        s += buf;
        s += head + consts;
        s += "    u64 ir_vis_ = 0;\n" + rej_decl(nck);
        s += "    for (u64 ir_p_ = ir_w0_; ir_p_ < ir_npar_; ir_p_ += ir_nw_) {\n" + parent;
        s += "        ir_vis_ += ir_n_;\n        u64 ir_c_ = 0;\n";
        s += "        for (u64 ir_i_ = ir_lane_; ir_i_ < ir_n_; ir_i_ += 32) {\n" + point;
        if (nck) s += rej_inc(nck, "            ");
        else s += "            ++ir_c_;\n";
        s += "        }\n        ir_c_ = warp_sum(ir_c_);\n        if (ir_lane_ == 0) ir_cnt_[ir_p_] = ir_c_;\n    }\n";
        snprintf(buf, sizeof(buf), "    if (ir_lane_ == 0 && ir_vis_) atomicAdd(&ir_stats_[%d], ir_vis_);\n", k);
        s += buf;
        for (int l = 0; l < nck; ++l) {
            snprintf(buf, sizeof(buf),
                     "    { const u64 ir_x_ = warp_sum(ir_rej%d_); if (ir_lane_ == 0 && ir_x_) atomicAdd(&ir_stats_[NI + %d], ir_x_); }\n",
                     l, idx[l]);
            s += buf;
        }
        s += "}\n";
        // emit
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_emit_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "const u64 *ir_off_, i64 *ir_out_) {\n", k);
        s += buf;
        s += head + consts;
        s += "    for (u64 ir_p_ = ir_w0_; ir_p_ < ir_npar_; ir_p_ += ir_nw_) {\n" + parent;
        s += "        u64 ir_pos_ = ir_off_[ir_p_];\n        if (ir_off_[ir_p_ + 1] == ir_pos_) continue;   // no children: nothing to re-evaluate\n";
        s += "        for (u64 ir_b_ = 0; ir_b_ < ir_n_; ir_b_ += 32) {\n";
        s += "            const u64 ir_i_ = ir_b_ + ir_lane_;\n            bool ir_keep_ = false;\n";
        s += "            if (ir_i_ < ir_n_) {\n" + point + "            ir_keep_ = ir_r_ == 0;\n            }\n";
        // the row: the parent's values + this level's value
        s += "            const unsigned ir_bal_ = __ballot_sync(0xffffffffu, ir_keep_);\n";
        s += "            if (ir_keep_) {\n";
        snprintf(buf, sizeof(buf),
                 "                i64 *ir_row_ = ir_out_ + (ir_pos_ + __popc(ir_bal_ & ((1u << ir_lane_) - 1u))) * %du;\n",
                 k + 1);
        s += buf;
        for (int j = 0; j < k; ++j) {
            snprintf(buf, sizeof(buf), "                ir_row_[%d] = ir_par_[ir_p_ * %d + %d];\n", j, k, j);
            s += buf;
        }
        snprintf(buf, sizeof(buf), "                ir_row_[%d] = ir_lo_ + (i64)ir_i_ * ir_st_;\n", k);
        s += buf;
        s += "            }\n            ir_pos_ += __popc(ir_bal_);\n        }\n    }\n}\n";
        // thread-per-parent variants (many parents with short ranges: a warp
        // per parent would leave most lanes idle and repeat the parent's
        // bindings 32 times)
        const std::string thead =
            "    const unsigned ir_lane_ = threadIdx.x & 31;\n"
            "    const u64 ir_t0_ = (u64)blockIdx.x * blockDim.x + threadIdx.x;\n"
            "    const u64 ir_nt_ = (u64)gridDim.x * blockDim.x;\n";
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_tcount_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "u64 *ir_cnt_, u64 *ir_stats_) {\n", k);
        s += buf;
        s += thead + consts;
        s += "    u64 ir_vis_ = 0;\n" + rej_decl(nck);
        s += "    for (u64 ir_p_ = ir_t0_; ir_p_ < ir_npar_; ir_p_ += ir_nt_) {\n" + parent;
        s += "        ir_vis_ += ir_n_;\n        u64 ir_c_ = 0;\n";
        s += "        for (u64 ir_i_ = 0; ir_i_ < ir_n_; ++ir_i_) {\n" + point;
        if (nck) s += rej_inc(nck, "            ");
        else s += "            ++ir_c_;\n";
        s += "        }\n        ir_cnt_[ir_p_] = ir_c_;\n    }\n";
        snprintf(buf, sizeof(buf), "    ir_vis_ = warp_sum(ir_vis_);\n    if (ir_lane_ == 0 && ir_vis_) atomicAdd(&ir_stats_[%d], ir_vis_);\n", k);
        s += buf;
        for (int l = 0; l < nck; ++l) {
            snprintf(buf, sizeof(buf),
                     "    { const u64 ir_x_ = warp_sum(ir_rej%d_); if (ir_lane_ == 0 && ir_x_) atomicAdd(&ir_stats_[NI + %d], ir_x_); }\n",
                     l, idx[l]);
            s += buf;
        }
        s += "}\n";
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_temit_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "const u64 *ir_off_, i64 *ir_out_) {\n", k);
        s += buf;
        s += thead + consts + "    (void)ir_lane_;\n";
        s += "    for (u64 ir_p_ = ir_t0_; ir_p_ < ir_npar_; ir_p_ += ir_nt_) {\n" + parent;
        s += "        u64 ir_pos_ = ir_off_[ir_p_];\n        if (ir_off_[ir_p_ + 1] == ir_pos_) continue;   // no children: nothing to re-evaluate\n";
        s += "        for (u64 ir_i_ = 0; ir_i_ < ir_n_; ++ir_i_) {\n" + point;
        s += "            if (ir_r_ == 0) {\n";
        snprintf(buf, sizeof(buf), "                i64 *ir_row_ = ir_out_ + ir_pos_ * %du;\n", k + 1);
        s += buf;
        for (int j = 0; j < k; ++j) {
            snprintf(buf, sizeof(buf), "                ir_row_[%d] = %s;\n", j, ir->inames[j].c_str());
            s += buf;
        }
        snprintf(buf, sizeof(buf), "                ir_row_[%d] = %s;\n                ++ir_pos_;\n", k,
                 ir->inames[k].c_str());
        s += buf;
        s += "            }\n        }\n    }\n}\n";

    }
    // Fused pairs (k, k + 1) for a level k without constraints: one thread per
    // parent runs both loops (the level-(k+1) range re-evaluated per value of
    // k), so the level-k rows are never materialised -- the engine takes them
    // when a level without constraints has many parents.
    for (int k = 0; k + 1 < ir->ni; ++k) {
        bool free_k = true;
        for (size_t j = 0; j < ir->kexpr.size(); ++j) free_k = free_k && ir->klev[j] != k;
        if (!free_k) continue;
        std::vector<int> idx;
        const std::string cons = constraints_at(k + 1, "                ", &idx);
        const int nck = (int)idx.size();
        std::string parent;
        for (int j = 0; j < k; ++j) {
            snprintf(buf, sizeof(buf), "        const i64 %s = ir_par_[ir_p_ * %d + %d]; (void)%s;\n",
                     ir->inames[j].c_str(), k, j, ir->inames[j].c_str());
            parent += buf;
        }
        parent += derived_at(-1, k - 1, "        ");
        parent += "        const i64 ir_lo_ = (i64)(" + ir->istart[k] + "), ir_hi_ = (i64)(" + ir->istop[k] +
                  "), ir_st_ = (i64)(" + ir->istep[k] + ");\n";
        parent += "        const u64 ir_n_ = ir_st_ == 0 ? 0ull : ir_trip(ir_lo_, ir_hi_, ir_st_);\n";
        std::string outer;   // value of k, its derived variables, the range of k + 1
        outer += "            const i64 " + ir->inames[k] + " = ir_lo_ + (i64)ir_i_ * ir_st_; (void)" +
                 ir->inames[k] + ";\n";
        outer += derived_at(k, k, "            ");
        outer += "            const i64 ir_lo2_ = (i64)(" + ir->istart[k + 1] + "), ir_hi2_ = (i64)(" +
                 ir->istop[k + 1] + "), ir_st2_ = (i64)(" + ir->istep[k + 1] + ");\n";
        outer += "            const u64 ir_n2_ = ir_st2_ == 0 ? 0ull : ir_trip(ir_lo2_, ir_hi2_, ir_st2_);\n";
        std::string inner;
        inner += "                const i64 " + ir->inames[k + 1] + " = ir_lo2_ + (i64)ir_j_ * ir_st2_; (void)" +
                 ir->inames[k + 1] + ";\n";
        inner += derived_at(k + 1, k + 1, "                ");
        inner += "                int ir_r_ = 0;\n" + cons;
        const std::string thead =
            "    const unsigned ir_lane_ = threadIdx.x & 31;\n"
            "    const u64 ir_t0_ = (u64)blockIdx.x * blockDim.x + threadIdx.x;\n"
            "    const u64 ir_nt_ = (u64)gridDim.x * blockDim.x;\n";
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_fcount_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "u64 *ir_cnt_, u64 *ir_stats_) {\n", k);
        s += buf;
        s += thead + consts;
        s += "    u64 ir_vis_ = 0, ir_vis2_ = 0;\n" + rej_decl(nck);
        s += "    for (u64 ir_p_ = ir_t0_; ir_p_ < ir_npar_; ir_p_ += ir_nt_) {\n" + parent;
        s += "        ir_vis_ += ir_n_;\n        u64 ir_c_ = 0;\n";
        s += "        for (u64 ir_i_ = 0; ir_i_ < ir_n_; ++ir_i_) {\n" + outer;
        s += "            ir_vis2_ += ir_n2_;\n";
        s += "            for (u64 ir_j_ = 0; ir_j_ < ir_n2_; ++ir_j_) {\n" + inner;
        if (nck) s += rej_inc(nck, "                ");
        else s += "                ++ir_c_;\n";
        s += "            }\n        }\n        ir_cnt_[ir_p_] = ir_c_;\n    }\n";
        snprintf(buf, sizeof(buf),
                 "    ir_vis_ = warp_sum(ir_vis_);\n    if (ir_lane_ == 0 && ir_vis_) atomicAdd(&ir_stats_[%d], ir_vis_);\n"
                 "    ir_vis2_ = warp_sum(ir_vis2_);\n    if (ir_lane_ == 0 && ir_vis2_) atomicAdd(&ir_stats_[%d], ir_vis2_);\n",
                 k, k + 1);
        s += buf;
        for (int l = 0; l < nck; ++l) {
            snprintf(buf, sizeof(buf),
                     "    { const u64 ir_x_ = warp_sum(ir_rej%d_); if (ir_lane_ == 0 && ir_x_) atomicAdd(&ir_stats_[NI + %d], ir_x_); }\n",
                     l, idx[l]);
            s += buf;
        }
        s += "}\n";
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_femit_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "const u64 *ir_off_, i64 *ir_out_) {\n", k);
        s += buf;
        s += thead + consts + "    (void)ir_lane_;\n";
        s += "    for (u64 ir_p_ = ir_t0_; ir_p_ < ir_npar_; ir_p_ += ir_nt_) {\n" + parent;
        s += "        u64 ir_pos_ = ir_off_[ir_p_];\n        if (ir_off_[ir_p_ + 1] == ir_pos_) continue;   // no children: nothing to re-evaluate\n";
        s += "        for (u64 ir_i_ = 0; ir_i_ < ir_n_; ++ir_i_) {\n" + outer;
        s += "            for (u64 ir_j_ = 0; ir_j_ < ir_n2_; ++ir_j_) {\n" + inner;
        s += "                if (ir_r_ == 0) {\n";
        snprintf(buf, sizeof(buf), "                    i64 *ir_row_ = ir_out_ + ir_pos_ * %du;\n", k + 2);
        s += buf;
        for (int j = 0; j <= k + 1; ++j) {
            snprintf(buf, sizeof(buf), "                    ir_row_[%d] = %s;\n", j, ir->inames[j].c_str());
            s += buf;
        }
        s += "                    ++ir_pos_;\n                }\n            }\n        }\n    }\n}\n";
        // warp-per-parent fused pair: lanes take the level-k values, each
        // lane runs the level-(k+1) loop of its value (uniform trip counts
        // when the inner range does not depend on the outer value)
        const std::string whead =
            "    const unsigned ir_lane_ = threadIdx.x & 31;\n"
            "    const u64 ir_w0_ = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;\n"
            "    const u64 ir_nw_ = ((u64)gridDim.x * blockDim.x) >> 5;\n";
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_wfcount_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "u64 *ir_cnt_, u64 *ir_stats_) {\n", k);
        s += buf;
        s += whead + consts;
        s += "    u64 ir_vis_ = 0, ir_vis2_ = 0;\n" + rej_decl(nck);
        // per parent, warp-uniform: lanes over the level-k values, or -- when
        // there are fewer than 32 of them and the level-(k+1) range of the
        // first one fills the lanes better -- the level-k values one after
        // another with the lanes over level k+1
        const std::string choose =
            "        bool ir_inner_ = false;\n"
            "        if (ir_n_ > 0 && ir_n_ < 32) {\n            const u64 ir_i_ = 0;\n" + outer +
            "            ir_inner_ = ir_n2_ * 32ull * ((ir_n_ + 31) / 32) > ir_n_ * 32ull * ((ir_n2_ + 31) / 32);\n"
            "        }\n";
        s += "    for (u64 ir_p_ = ir_w0_; ir_p_ < ir_npar_; ir_p_ += ir_nw_) {\n" + parent + choose;
        s += "        ir_vis_ += ir_n_;\n        u64 ir_c_ = 0;\n";
        s += "        if (!ir_inner_) {\n";
        s += "        for (u64 ir_i_ = ir_lane_; ir_i_ < ir_n_; ir_i_ += 32) {\n" + outer;
        s += "            ir_vis2_ += ir_n2_;\n";
        s += "            for (u64 ir_j_ = 0; ir_j_ < ir_n2_; ++ir_j_) {\n" + inner;
        if (nck) s += rej_inc(nck, "                ");
        else s += "                ++ir_c_;\n";
        s += "            }\n        }\n        } else {\n";
        s += "        for (u64 ir_i_ = 0; ir_i_ < ir_n_; ++ir_i_) {\n" + outer;
        s += "            if (ir_lane_ == 0) ir_vis2_ += ir_n2_;\n";
        s += "            for (u64 ir_j_ = ir_lane_; ir_j_ < ir_n2_; ir_j_ += 32) {\n" + inner;
        if (nck) s += rej_inc(nck, "                ");
        else s += "                ++ir_c_;\n";
        s += "            }\n        }\n        }\n";
        s += "        ir_c_ = warp_sum(ir_c_);\n        if (ir_lane_ == 0) ir_cnt_[ir_p_] = ir_c_;\n    }\n";
        snprintf(buf, sizeof(buf),
                 "    if (ir_lane_ == 0 && ir_vis_) atomicAdd(&ir_stats_[%d], ir_vis_);\n"
                 "    ir_vis2_ = warp_sum(ir_vis2_);\n    if (ir_lane_ == 0 && ir_vis2_) atomicAdd(&ir_stats_[%d], ir_vis2_);\n",
                 k, k + 1);
        s += buf;
        for (int l = 0; l < nck; ++l) {
            snprintf(buf, sizeof(buf),
                     "    { const u64 ir_x_ = warp_sum(ir_rej%d_); if (ir_lane_ == 0 && ir_x_) atomicAdd(&ir_stats_[NI + %d], ir_x_); }\n",
                     l, idx[l]);
            s += buf;
        }
        s += "}\n";
        snprintf(buf, sizeof(buf),
                 "extern \"C\" __global__ void __launch_bounds__(256) ir_wfemit_%d(const i64 *ir_par_, u64 ir_npar_, "
                 "const u64 *ir_off_, i64 *ir_out_) {\n", k);
        s += buf;
        s += whead + consts;
        s += "    for (u64 ir_p_ = ir_w0_; ir_p_ < ir_npar_; ir_p_ += ir_nw_) {\n" + parent + choose;
        s += "        u64 ir_pos_ = ir_off_[ir_p_];\n        if (ir_off_[ir_p_ + 1] == ir_pos_) continue;   // no children: nothing to re-evaluate\n";
        // lanes over level k+1: ballot-ranked rows, value by value
        s += "        if (ir_inner_) {\n";
        s += "        for (u64 ir_i_ = 0; ir_i_ < ir_n_; ++ir_i_) {\n" + outer;
        s += "            for (u64 ir_jb_ = 0; ir_jb_ < ir_n2_; ir_jb_ += 32) {\n";
        s += "                const u64 ir_j_ = ir_jb_ + ir_lane_;\n                bool ir_keep_ = false;\n";
        s += "                if (ir_j_ < ir_n2_) {\n" + inner + "                ir_keep_ = ir_r_ == 0;\n                }\n";
        s += "                const unsigned ir_bal_ = __ballot_sync(0xffffffffu, ir_keep_);\n";
        s += "                if (ir_keep_) {\n";
        snprintf(buf, sizeof(buf),
                 "                    i64 *ir_row_ = ir_out_ + (ir_pos_ + __popc(ir_bal_ & ((1u << ir_lane_) - 1u))) * %du;\n",
                 k + 2);
        s += buf;
        for (int j = 0; j <= k; ++j) {
            snprintf(buf, sizeof(buf), "                    ir_row_[%d] = %s;\n", j, ir->inames[j].c_str());
            s += buf;
        }
        snprintf(buf, sizeof(buf), "                    ir_row_[%d] = ir_lo2_ + (i64)ir_j_ * ir_st2_;\n", k + 1);
        s += buf;
        s += "                }\n                ir_pos_ += __popc(ir_bal_);\n            }\n        }\n        continue;\n        }\n";
        s += "        for (u64 ir_b_ = 0; ir_b_ < ir_n_; ir_b_ += 32) {\n";
        s += "            const u64 ir_i_ = ir_b_ + ir_lane_;\n            u64 ir_k_ = 0;\n";
        s += "            if (ir_i_ < ir_n_) {\n" + outer;
        s += "            for (u64 ir_j_ = 0; ir_j_ < ir_n2_; ++ir_j_) {\n" + inner;
        s += "                if (ir_r_ == 0) ++ir_k_;\n            }\n            }\n";
        // warp exclusive scan of the lanes' survivor counts (lane order = value order of level k)
        s += "            u64 ir_x_ = ir_k_;\n";
        s += "            for (int ir_o_ = 1; ir_o_ < 32; ir_o_ <<= 1) { const u64 ir_y_ = __shfl_up_sync(0xffffffffu, ir_x_, ir_o_); if ((int)ir_lane_ >= ir_o_) ir_x_ += ir_y_; }\n";
        s += "            const u64 ir_tot_ = __shfl_sync(0xffffffffu, ir_x_, 31);\n";
        s += "            if (ir_k_) {\n                u64 ir_q_ = ir_pos_ + ir_x_ - ir_k_;\n" + outer;
        s += "            for (u64 ir_j_ = 0; ir_j_ < ir_n2_; ++ir_j_) {\n" + inner;
        s += "                if (ir_r_ == 0) {\n";
        snprintf(buf, sizeof(buf), "                    i64 *ir_row_ = ir_out_ + ir_q_ * %du;\n", k + 2);
        s += buf;
        for (int j = 0; j <= k + 1; ++j) {
            snprintf(buf, sizeof(buf), "                    ir_row_[%d] = %s;\n", j, ir->inames[j].c_str());
            s += buf;
        }
        s += "                    ++ir_q_;\n                }\n            }\n            }\n";
        s += "            ir_pos_ += ir_tot_;\n        }\n    }\n}\n";
    }
    return s;
}

int compile_load(beast_ir *ir) {
    Nvrtc &n = nvrtc();
    if (!n.ok) {
        ir->err = "libnvrtc could not be loaded (set BEAST_NVRTC to its path)";
        return BEAST_ERR_UNSUPPORTED;
    }
    nvrtcProgram_t prog = nullptr;
    if (n.create(&prog, ir->src.c_str(), "beast_ir.cu", 0, nullptr, nullptr) != 0) {
        ir->err = "nvrtcCreateProgram failed";
        return BEAST_ERR_UNSUPPORTED;
    }
    const char *opts[] = {"-arch=sm_100a", "-std=c++17", "-lineinfo"};
    const int rc = n.compile(prog, 3, opts);
    size_t ls = 0;
    n.log_size(prog, &ls);
    std::string log(ls, '\0');
    if (ls) n.log(prog, &log[0]);
    if (rc != 0) {
        ir->err = "NVRTC compile failed: " + log.substr(0, 2000);
        n.destroy(&prog);
        return BEAST_ERR_INVALID_ARGUMENT;
    }
    size_t cs = 0;
    n.cubin_size(prog, &cs);
    ir->cubin.resize(cs);
    n.cubin(prog, ir->cubin.data());
    n.destroy(&prog);
    return BEAST_OK;
}

int load(beast_ir *ir) {
    if (ir->lib) return BEAST_OK;
    IRCK(cudaGetDevice(&ir->device));
    IRCK(cudaDeviceGetAttribute(&ir->sm_count, cudaDevAttrMultiProcessorCount, ir->device));
    IRCK(cudaLibraryLoadData(&ir->lib, ir->cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0));
    {
        // the level buffers are stream-ordered allocations from the device's
        // default pool: keep them mapped between runs (the default release
        // threshold of 0 would unmap and re-map gigabytes on every call)
        cudaMemPool_t pool;
        IRCK(cudaDeviceGetDefaultMemPool(&pool, ir->device));
        unsigned long long keep = ~0ull;
        IRCK(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep));
    }
    IRCK(cudaLibraryGetKernel(&ir->k_root, ir->lib, "ir_root"));
    ir->k_count.assign(ir->ni, nullptr);
    ir->k_emit.assign(ir->ni, nullptr);
    ir->k_tcount.assign(ir->ni, nullptr);
    ir->k_temit.assign(ir->ni, nullptr);
    for (int k = 0; k < ir->ni; ++k) {
        IRCK(cudaLibraryGetKernel(&ir->k_count[k], ir->lib, ("ir_count_" + std::to_string(k)).c_str()));
        IRCK(cudaLibraryGetKernel(&ir->k_emit[k], ir->lib, ("ir_emit_" + std::to_string(k)).c_str()));
        IRCK(cudaLibraryGetKernel(&ir->k_tcount[k], ir->lib, ("ir_tcount_" + std::to_string(k)).c_str()));
        IRCK(cudaLibraryGetKernel(&ir->k_temit[k], ir->lib, ("ir_temit_" + std::to_string(k)).c_str()));
    }
    ir->k_fcount.assign(ir->ni, nullptr);
    ir->k_femit.assign(ir->ni, nullptr);
    ir->k_wfcount.assign(ir->ni, nullptr);
    ir->k_wfemit.assign(ir->ni, nullptr);
    for (int k = 0; k + 1 < ir->ni; ++k) {
        // fuse (k, k + 1) where level k has no constraints and level k + 1
        // filters (or is the deepest): its rows are the ones materialised
        bool free_k = true, filters = k + 2 == ir->ni;
        for (size_t j = 0; j < ir->kexpr.size(); ++j) {
            free_k = free_k && ir->klev[j] != k;
            filters = filters || ir->klev[j] == k + 1;
        }
        if (!free_k || !filters) continue;
        IRCK(cudaLibraryGetKernel(&ir->k_fcount[k], ir->lib, ("ir_fcount_" + std::to_string(k)).c_str()));
        IRCK(cudaLibraryGetKernel(&ir->k_femit[k], ir->lib, ("ir_femit_" + std::to_string(k)).c_str()));
        IRCK(cudaLibraryGetKernel(&ir->k_wfcount[k], ir->lib, ("ir_wfcount_" + std::to_string(k)).c_str()));
        IRCK(cudaLibraryGetKernel(&ir->k_wfemit[k], ir->lib, ("ir_wfemit_" + std::to_string(k)).c_str()));
    }
    IRCK(cudaLibraryGetKernel(&ir->k_tiles, ir->lib, "ir_scan_tiles"));
    IRCK(cudaLibraryGetKernel(&ir->k_top, ir->lib, "ir_scan_top"));
    IRCK(cudaLibraryGetKernel(&ir->k_add, ir->lib, "ir_scan_add"));
    return BEAST_OK;
}

int launch(beast_ir *ir, cudaKernel_t k, unsigned grid, unsigned block, cudaStream_t st, void **args) {
    IRCK(cudaLaunchKernel((const void *)k, dim3(grid), dim3(block), args, 0, st));
    return BEAST_OK;
}

// Exclusive scan of n u64 counts into off[0..n] (off[n] = total); returns the total (host).
// total == nullptr: no host copy and no synchronisation (the device total
// is written to tot_dev).
int scan(beast_ir *ir, const unsigned long long *cnt, unsigned long long n, unsigned long long *off,
         cudaStream_t st, unsigned long long *total, unsigned long long *tot_dev) {
    const unsigned long long tiles = std::max(1ull, (n + 2047) / 2048);
    unsigned long long *ts = nullptr, *tot = nullptr;
    IRCK(cudaMallocAsync((void **)&ts, (tiles + 1) * 8, st));
    tot = ts + tiles;
    {
        void *a[] = {(void *)&cnt, (void *)&n, (void *)&off, (void *)&ts};
        if (launch(ir, ir->k_tiles, (unsigned)tiles, 256, st, a) != BEAST_OK) return BEAST_ERR_CUDA;
    }
    {
        unsigned long long nt = tiles;
        void *a[] = {(void *)&ts, (void *)&nt, (void *)&tot};
        if (launch(ir, ir->k_top, 1, 1024, st, a) != BEAST_OK) return BEAST_ERR_CUDA;
    }
    {
        const unsigned g = (unsigned)std::max(1ull, (n + 255) / 256);
        void *a[] = {(void *)&off, (void *)&n, (void *)&ts, (void *)&tot};
        if (launch(ir, ir->k_add, g, 256, st, a) != BEAST_OK) return BEAST_ERR_CUDA;
    }
    if (tot_dev) IRCK(cudaMemcpyAsync(tot_dev, tot, 8, cudaMemcpyDeviceToDevice, st));
    if (total) IRCK(cudaMemcpyAsync(total, tot, 8, cudaMemcpyDeviceToHost, st));
    IRCK(cudaFreeAsync(ts, st));
    if (total) IRCK(cudaStreamSynchronize(st));
    return BEAST_OK;
}

int run(beast_ir *ir, cudaStream_t st, long long *out, unsigned long long capacity, unsigned long long *written,
        unsigned long long *visits, unsigned long long *rejected, bool emit_last, bool allow_replay = true) {
    const int lrc = load(ir);
    if (lrc != BEAST_OK) return lrc;
    int dev = 0;
    IRCK(cudaGetDevice(&dev));
    if (dev != ir->device) {
        ir->err = "IR compiled for another device";
        return BEAST_ERR_INVALID_ARGUMENT;
    }
    const int NI = ir->ni, NC = ir->nc;
    unsigned long long *stats = nullptr;
    int *pruned_d = nullptr;
    IRCK(cudaMallocAsync((void **)&stats, (size_t)(NI + NC + 1 + 2 * NI + 1) * 8, st));
    IRCK(cudaMemsetAsync(stats, 0, (size_t)(NI + NC + 1) * 8, st));
    pruned_d = (int *)(stats + NI + NC);
    unsigned long long *trip_d = stats + NI + NC + 1;   // static trip count per iterator (~0: depends on the parent)
    unsigned long long *tot_d = trip_d + NI;             // device total of each step's deepest level
    if (NI) IRCK(cudaMemsetAsync(tot_d, 0xff, (size_t)NI * 8, st));
    {
        void *a[] = {(void *)&stats, (void *)&pruned_d, (void *)&trip_d};
        if (launch(ir, ir->k_root, 1, 1, st, a) != BEAST_OK) return BEAST_ERR_CUDA;
    }
    // replay: the previous run's totals stand in for the per-level host
    // round trips (BEAST_IR_TRACE and the first run synchronise per level)
    const bool trace_env = getenv("BEAST_IR_TRACE") != nullptr;
    const bool replay = !trace_env && allow_replay && ir->known_pruned >= 0 && (int)ir->known_tot.size() == NI;
    int pruned = 0;
    std::vector<unsigned long long> trip(NI + 1, ~0ull);
    if (replay) {
        pruned = ir->known_pruned;
        for (int k = 0; k < NI; ++k) trip[k] = ir->known_trip[k];
    } else {
        IRCK(cudaMemcpyAsync(&pruned, pruned_d, sizeof(int), cudaMemcpyDeviceToHost, st));
        if (NI) IRCK(cudaMemcpyAsync(trip.data(), trip_d, (size_t)NI * 8, cudaMemcpyDeviceToHost, st));
        IRCK(cudaStreamSynchronize(st));
    }
    std::vector<unsigned long long> step_tot(NI, ~0ull);   // host totals of this run's steps (recording runs)
    unsigned long long n_par = pruned ? 0 : 1;
    long long *par = nullptr;   // level -1: one empty tuple
    int rc = BEAST_OK;
    unsigned long long total = 0;
    const unsigned grid = (unsigned)ir->sm_count * 8;
    // thread per parent once the parents outnumber the resident threads many
    // times over (BEAST_IR_THREAD_MIN, default 64 x 8 CTAs x 256 threads per SM)
    unsigned long long thread_min = 64ull * grid * 256;
    if (const char *e = getenv("BEAST_IR_THREAD_MIN")) thread_min = strtoull(e, nullptr, 10);

    // levels k, k + 1 fused (level k has no constraints) once level k has
    // this many parents (BEAST_IR_FUSE_MIN, default 8 x 8 CTAs x 256 threads per SM)
    unsigned long long fuse_min = 8ull * grid * 256;
    if (const char *e = getenv("BEAST_IR_FUSE_MIN")) fuse_min = strtoull(e, nullptr, 10);
    // BEAST_IR_TRACE=1: per-level step time and shape on stderr (development)
    const bool trace = getenv("BEAST_IR_TRACE") != nullptr;
    cudaEvent_t tev[2] = {nullptr, nullptr};
    if (trace) {
        cudaEventCreate(&tev[0]);
        cudaEventCreate(&tev[1]);
    }
    if ((int)ir->avg_trip.size() != NI) ir->avg_trip.assign(NI, -1.0);
    if ((int)ir->fuse_known.size() != NI) ir->fuse_known.assign(NI, -1);
    std::vector<unsigned long long> step_par(NI, 0);   // parents of the levels that start a step
    for (int k = 0; k < NI && n_par;) {
        if (trace) cudaEventRecord(tev[0], st);
        const unsigned long long n_par_in = n_par;
        step_par[k] = n_par;
        bool fused = ir->k_fcount[k] != nullptr && n_par >= fuse_min;
        if (!fused && ir->k_fcount[k] != nullptr && ir->fuse_known[k] >= 0) fused = ir->fuse_known[k] == 1;
        // thread per parent: very many parents, or a level whose (constant)
        // trip count is so short that a warp per parent would idle most lanes
        // (BEAST_IR_SHORT_TRIP, default 8), given enough parents to fill the GPU
        unsigned long long short_trip = 8;
        if (const char *e = getenv("BEAST_IR_SHORT_TRIP")) short_trip = strtoull(e, nullptr, 10);
        // the trip count: constant, else the previous run's average
        const double trip_est = trip[k] != ~0ull ? (double)trip[k] : ir->avg_trip[k];
        const bool short_level = ir->k_fcount[k] == nullptr || !fused;   // (a fused step runs two loops)
        const bool tmode = n_par >= thread_min ||
                           (short_level && trip_est >= 0 && trip_est <= (double)short_trip &&
                            n_par >= (unsigned long long)grid * 256);

        if (!fused && ir->k_fcount[k] != nullptr && ir->fuse_known[k] < 0) {
            // would level k's rows be large?  count them (level k has no
            // constraints: the children are its trip counts) and fuse with
            // k + 1 instead of materialising more than BEAST_IR_MATERIALIZE_MAX
            // bytes (default 64 MiB)
            unsigned long long lim = 64ull << 20;
            if (const char *e = getenv("BEAST_IR_MATERIALIZE_MAX")) lim = strtoull(e, nullptr, 10);
            unsigned long long *cnt0 = nullptr, *stats0 = nullptr;
            IRCK(cudaMallocAsync((void **)&cnt0, (n_par + 1) * 8, st));
            IRCK(cudaMallocAsync((void **)&stats0, (size_t)(NI + NC + 1) * 8, st));   // scratch statistics
            const long long *pc = par;
            void *a[] = {(void *)&pc, (void *)&n_par, (void *)&cnt0, (void *)&stats0};
            rc = launch(ir, tmode ? ir->k_tcount[k] : ir->k_count[k], grid, 256, st, a);
            unsigned long long *off0 = nullptr, kids = 0;
            if (rc == BEAST_OK) IRCK(cudaMallocAsync((void **)&off0, (n_par + 1) * 8, st));
            if (rc == BEAST_OK) rc = scan(ir, cnt0, n_par, off0, st, &kids, nullptr);
            cudaFreeAsync(cnt0, st);
            cudaFreeAsync(stats0, st);
            if (off0) cudaFreeAsync(off0, st);
            if (rc != BEAST_OK) break;
            fused = kids * (unsigned long long)(k + 1) * 8 > lim;
            ir->fuse_known[k] = fused ? 1 : 0;
        }
        const bool wfused = fused && !tmode;   // warp per parent unless there are very many parents
        const int k_last = fused ? k + 1 : k;   // deepest level of this step
        unsigned long long *cnt = nullptr, *off = nullptr;
        IRCK(cudaMallocAsync((void **)&cnt, (n_par + 1) * 8, st));
        IRCK(cudaMallocAsync((void **)&off, (n_par + 1) * 8, st));
        {
            const long long *pc = par;
            void *a[] = {(void *)&pc, (void *)&n_par, (void *)&cnt, (void *)&stats};
            rc = launch(ir, wfused ? ir->k_wfcount[k] : fused ? ir->k_fcount[k] : tmode ? ir->k_tcount[k] : ir->k_count[k],
                        grid, 256, st, a);
        }
        const bool replay_step = replay && ir->known_tot[k_last] != ~0ull;
        if (rc == BEAST_OK) rc = scan(ir, cnt, n_par, off, st, replay_step ? nullptr : &total, tot_d + k_last);
        if (replay_step) total = ir->known_tot[k_last];
        else step_tot[k_last] = total;
        long long *child = nullptr;
        const bool last = k_last == NI - 1;
        if (rc == BEAST_OK && (!last || emit_last) && total) {
            if (last) {
                if (total > capacity) rc = BEAST_ERR_CAPACITY;
                else child = out;
            } else {
                const cudaError_t e = cudaMallocAsync((void **)&child, total * (unsigned long long)(k_last + 1) * 8, st);
                if (e != cudaSuccess) {
                    ir->err = "out of device memory for level " + std::to_string(k_last) + " (" + std::to_string(total) +
                              " tuples)";
                    rc = BEAST_ERR_WORKSPACE;
                }
            }
            if (rc == BEAST_OK) {
                const long long *pc = par;
                void *a[] = {(void *)&pc, (void *)&n_par, (void *)&off, (void *)&child};
                rc = launch(ir, wfused ? ir->k_wfemit[k] : fused ? ir->k_femit[k] : tmode ? ir->k_temit[k] : ir->k_emit[k],
                            grid, 256, st, a);
            }
        }
        cudaFreeAsync(cnt, st);
        cudaFreeAsync(off, st);
        if (par) cudaFreeAsync(par, st);
        par = (last || rc != BEAST_OK) ? nullptr : child;
        n_par = total;
        if (trace) {
            float ms = 0;
            cudaEventRecord(tev[1], st);
            cudaEventSynchronize(tev[1]);
            cudaEventElapsedTime(&ms, tev[0], tev[1]);
            fprintf(stderr, "ir level %d%s%s: parents %llu -> children %llu  %.4f ms\n", k, fused ? "+1 (fused)" : "",
                    tmode ? " thread/parent" : " warp/parent", n_par_in, total, ms);
        }
        if (rc != BEAST_OK) {
            if (child && child != out) cudaFreeAsync(child, st);
            break;
        }
        k = k_last + 1;
    }
    if (trace) {
        cudaEventDestroy(tev[0]);
        cudaEventDestroy(tev[1]);
    }
    if (NI == 0) total = pruned ? 0 : 1;
    std::vector<unsigned long long> h(NI + NC), dtot(NI, ~0ull);
    if (NI + NC) IRCK(cudaMemcpyAsync(h.data(), stats, (size_t)(NI + NC) * 8, cudaMemcpyDeviceToHost, st));
    if (NI) IRCK(cudaMemcpyAsync(dtot.data(), tot_d, (size_t)NI * 8, cudaMemcpyDeviceToHost, st));
    IRCK(cudaFreeAsync(stats, st));
    IRCK(cudaStreamSynchronize(st));
    if (replay) {
        // every replayed total must be what the device computed; otherwise
        // forget them and run again with a host round trip per level
        bool same = rc == BEAST_OK || rc == BEAST_ERR_CAPACITY;
        for (int k = 0; k < NI && same; ++k)
            if (dtot[k] != ~0ull && ir->known_tot[k] != ~0ull && dtot[k] != ir->known_tot[k]) same = false;
        if (!same) {
            ir->known_pruned = -1;
            ir->known_tot.clear();
            return run(ir, st, out, capacity, written, visits, rejected, emit_last, false);
        }
    } else if (rc == BEAST_OK) {
        if ((int)ir->known_tot.size() != NI) ir->known_tot.assign(NI, ~0ull);
        for (int k = 0; k < NI; ++k)
            if (step_tot[k] != ~0ull) ir->known_tot[k] = step_tot[k];
        ir->known_trip.assign(trip.begin(), trip.begin() + NI);
        ir->known_pruned = pruned;
    }
    if (rc != BEAST_OK && rc != BEAST_ERR_CAPACITY) return rc;
    if (rc == BEAST_OK)   // learn each step's trip counts for the next run
        for (int i = 0; i < NI; ++i)
            if (step_par[i]) ir->avg_trip[i] = (double)h[i] / (double)step_par[i];
    if (visits) for (int i = 0; i < NI; ++i) visits[i] = h[i];
    if (rejected) for (int i = 0; i < NC; ++i) rejected[i] = h[NI + i];
    if (written) *written = pruned ? 0 : total;
    return rc;
}

}  // namespace

extern "C" {

int beast_ir_create(const beast_ir_desc *d, beast_ir **out) {
    if (!d || !out) return BEAST_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    if (d->n_constants < 0 || d->n_iterators < 0 || d->n_derived < 0 || d->n_constraints < 0 ||
        d->n_iterators > 64 || d->n_constraints > 64)
        return BEAST_ERR_INVALID_ARGUMENT;
    auto *ir = new (std::nothrow) beast_ir();
    if (!ir) return BEAST_ERR_WORKSPACE;
    auto fail = [&](int rc) {
        *out = ir;   // handle kept so beast_ir_last_error can explain; caller destroys it
        return rc;
    };
    auto str = [](const char *s) { return std::string(s ? s : ""); };
    for (int i = 0; i < d->n_constants; ++i) {
        if (!valid_name(d->constant_names[i])) { ir->err = "bad constant name"; return fail(BEAST_ERR_INVALID_ARGUMENT); }
        ir->cnames.push_back(d->constant_names[i]);
        ir->cvals.push_back(d->constant_values[i]);
    }
    for (int i = 0; i < d->n_iterators; ++i) {
        if (!valid_name(d->iterator_names[i]) || !d->iterator_start[i] || !d->iterator_stop[i] ||
            !d->iterator_step[i]) {
            ir->err = "bad iterator " + std::to_string(i);
            return fail(BEAST_ERR_INVALID_ARGUMENT);
        }
        ir->inames.push_back(d->iterator_names[i]);
        ir->istart.push_back(str(d->iterator_start[i]));
        ir->istop.push_back(str(d->iterator_stop[i]));
        ir->istep.push_back(str(d->iterator_step[i]));
    }
    for (int i = 0; i < d->n_derived; ++i) {
        if (!valid_name(d->derived_names[i]) || !d->derived_exprs[i]) {
            ir->err = "bad derived variable " + std::to_string(i);
            return fail(BEAST_ERR_INVALID_ARGUMENT);
        }
        ir->dnames.push_back(d->derived_names[i]);
        ir->dexpr.push_back(str(d->derived_exprs[i]));
    }
    for (int i = 0; i < d->n_constraints; ++i) {
        if (!d->constraint_names[i] || !d->constraint_exprs[i]) {
            ir->err = "bad constraint " + std::to_string(i);
            return fail(BEAST_ERR_INVALID_ARGUMENT);
        }
        ir->knames.push_back(d->constraint_names[i]);
        ir->kexpr.push_back(str(d->constraint_exprs[i]));
    }
    ir->ni = d->n_iterators;
    ir->nc = d->n_constraints;
    int rc = analyse(ir);
    if (rc != BEAST_OK) return fail(rc);
    ir->src = generate(ir);
    rc = compile_load(ir);
    if (rc != BEAST_OK) return fail(rc);
    *out = ir;
    return BEAST_OK;
}

void beast_ir_destroy(beast_ir *ir) {
    if (!ir) return;
    if (ir->lib) cudaLibraryUnload(ir->lib);
    delete ir;
}

const char *beast_ir_last_error(const beast_ir *ir) { return ir ? ir->err.c_str() : "null handle"; }

const char *beast_ir_source(const beast_ir *ir) { return ir ? ir->src.c_str() : nullptr; }

int beast_ir_levels(const beast_ir *ir, int32_t *derived_levels, int32_t *constraint_levels) {
    if (!ir || ir->src.empty()) return BEAST_ERR_INVALID_ARGUMENT;
    if (derived_levels) for (size_t i = 0; i < ir->dlev.size(); ++i) derived_levels[i] = ir->dlev[i];
    if (constraint_levels) for (size_t i = 0; i < ir->klev.size(); ++i) constraint_levels[i] = ir->klev[i];
    return BEAST_OK;
}

int beast_ir_count(beast_ir *ir, void *stream, uint64_t *survivors, uint64_t *visits, uint64_t *rejected) {
    if (!ir || !survivors || ir->cubin.empty()) return BEAST_ERR_INVALID_ARGUMENT;
    unsigned long long n = 0;
    const int rc = run(ir, (cudaStream_t)stream, nullptr, 0, &n, (unsigned long long *)visits,
                       (unsigned long long *)rejected, false);
    if (rc == BEAST_OK) *survivors = n;
    return rc;
}

int beast_ir_enumerate(beast_ir *ir, void *stream, int64_t *out, uint64_t capacity, uint64_t *written,
                       uint64_t *visits, uint64_t *rejected) {
    if (!ir || !written || ir->cubin.empty() || (!out && capacity)) return BEAST_ERR_INVALID_ARGUMENT;
    unsigned long long n = 0;
    const int rc = run(ir, (cudaStream_t)stream, (long long *)out, capacity, &n, (unsigned long long *)visits,
                       (unsigned long long *)rejected, true);
    *written = n;
    return rc;
}

}  // extern "C"
