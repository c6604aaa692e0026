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
// Fixed text appended after the generated level functions.  ir_range(k, v)
// and ir_eval(k, v) read iterator values v[0..k] (v[k] = the candidate value
// for ir_eval); ir_eval returns 0 (passes level k) or 1 + the index of the
// first constraint of level k that holds.
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

// Constant-level constraints (no iterator): stats[NI + c] += 1 for the first
// one that holds; *pruned = 1 + c, or 0.
extern "C" __global__ void ir_root(u64 *stats, int *pruned) {
    const int r = ir_eval(-1, nullptr);
    *pruned = r;
    if (r) stats[NI + r - 1] += 1;
}

// One warp per parent tuple (rows of width k): number of children per parent
// into cnt[p]; visits of level k and first-failing rejections into stats.
extern "C" __global__ void __launch_bounds__(256) ir_count(int k, const i64 *par, u64 n_par, u64 *cnt, u64 *stats) {
    const unsigned lane = threadIdx.x & 31;
    const u64 w0 = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;
    u64 visits = 0, rej[NC > 0 ? NC : 1];
    for (int c = 0; c < NC; ++c) rej[c] = 0;
    i64 v[NI];
    for (u64 p = w0; p < n_par; p += nw) {
        for (int j = 0; j < k; ++j) v[j] = par[p * k + j];
        i64 lo, hi, st;
        ir_range(k, v, lo, hi, st);
        const u64 n = st == 0 ? 0ull : ir_trip(lo, hi, st);
        visits += n;
        u64 c = 0;
        for (u64 i = lane; i < n; i += 32) {
            v[k] = lo + (i64)i * st;
            const int r = ir_eval(k, v);
            if (r == 0) ++c;
            else rej[r - 1] += 1;
        }
        c = warp_sum(c);
        if (lane == 0) cnt[p] = c;
    }
    if (lane == 0 && visits) atomicAdd(&stats[k], visits);
    for (int c = 0; c < NC; ++c) {
        const u64 x = warp_sum(rej[c]);
        if (lane == 0 && x) atomicAdd(&stats[NI + c], x);
    }
}

// Emission: re-evaluate in order, write child rows (width k + 1) at
// off[p] + warp rank (canonical order).
extern "C" __global__ void __launch_bounds__(256) ir_emit(int k, const i64 *par, u64 n_par, const u64 *off, i64 *out) {
    const unsigned lane = threadIdx.x & 31;
    const u64 w0 = ((u64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const u64 nw = ((u64)gridDim.x * blockDim.x) >> 5;
    i64 v[NI];
    for (u64 p = w0; p < n_par; p += nw) {
        for (int j = 0; j < k; ++j) v[j] = par[p * k + j];
        i64 lo, hi, st;
        ir_range(k, v, lo, hi, st);
        const u64 n = st == 0 ? 0ull : ir_trip(lo, hi, st);
        u64 pos = off[p];
        for (u64 base = 0; base < n; base += 32) {
            const u64 i = base + lane;
            bool keep = false;
            if (i < n) {
                v[k] = lo + (i64)i * st;
                keep = ir_eval(k, v) == 0;
            }
            const unsigned b = __ballot_sync(0xffffffffu, keep);
            if (keep) {
                i64 *row = out + (pos + __popc(b & ((1u << lane) - 1u))) * (u64)(k + 1);
                for (int j = 0; j <= k; ++j) row[j] = v[j];
            }
            pos += __popc(b);
        }
    }
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
extern "C" __global__ void ir_scan_top(u64 *tile_sum, u64 n_tiles, u64 *total) {
    if (threadIdx.x != 0) return;
    u64 run = 0;
    for (u64 t = 0; t < n_tiles; ++t) { const u64 x = tile_sum[t]; tile_sum[t] = run; run += x; }
    *total = run;
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
    cudaKernel_t k_root = nullptr, k_count = nullptr, k_emit = nullptr, k_tiles = nullptr, k_top = nullptr,
                 k_add = nullptr;
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

std::string generate(const beast_ir *ir) {
    std::string s;
    char buf[256];
    s += "// generated by beast_ir_create (SURVEY §8(f) NEXT #4)\n";
    s += "typedef long long i64;\n";
    snprintf(buf, sizeof(buf), "#define NI %d\n#define NC %d\n", ir->ni, ir->nc);
    s += buf;
    auto consts = [&]() {
        std::string c;
        for (size_t i = 0; i < ir->cnames.size(); ++i) {
            snprintf(buf, sizeof(buf), "    const i64 %s = (i64)(%lldLL); (void)%s;\n", ir->cnames[i].c_str(),
                     ir->cvals[i], ir->cnames[i].c_str());
            c += buf;
        }
        return c;
    };
    // bindings visible at level k: iterators 0..k-1 (k_inclusive: 0..k), and
    // derived variables of level <= the deepest bound iterator, in order
    auto bind = [&](int upto) {   // iterators 0..upto bound
        std::string c;
        for (int j = 0; j <= upto; ++j) {
            snprintf(buf, sizeof(buf), "    const i64 %s = ir_v_[%d]; (void)%s;\n", ir->inames[j].c_str(), j,
                     ir->inames[j].c_str());
            c += buf;
        }
        for (size_t d = 0; d < ir->dnames.size(); ++d)
            if (ir->dlev[d] <= upto)
                c += "    const i64 " + ir->dnames[d] + " = (i64)(" + ir->dexpr[d] + "); (void)" + ir->dnames[d] + ";\n";
        return c;
    };
    s += "__device__ __forceinline__ void ir_range(int ir_k_, const i64 *ir_v_, i64 &ir_lo_, i64 &ir_hi_, "
         "i64 &ir_st_) {\n";
    s += "    (void)ir_v_;\n";
    s += "    switch (ir_k_) {\n";
    for (int k = 0; k < ir->ni; ++k) {
        snprintf(buf, sizeof(buf), "    case %d: {\n", k);
        s += buf;
        s += consts();
        s += bind(k - 1);
        s += "    ir_lo_ = (i64)(" + ir->istart[k] + "); ir_hi_ = (i64)(" + ir->istop[k] + "); ir_st_ = (i64)(" +
             ir->istep[k] + ");\n    return; }\n";
    }
    s += "    default: ir_lo_ = ir_hi_ = 0; ir_st_ = 1; return;\n    }\n}\n";
    s += "__device__ __forceinline__ int ir_eval(int ir_k_, const i64 *ir_v_) {\n";
    s += "    (void)ir_v_;\n";
    s += "    switch (ir_k_) {\n";
    for (int k = -1; k < ir->ni; ++k) {
        snprintf(buf, sizeof(buf), "    case %d: {\n", k);
        s += buf;
        s += consts();
        s += bind(k);
        for (size_t c = 0; c < ir->kexpr.size(); ++c)
            if (ir->klev[c] == k) {
                s += "    if ((" + ir->kexpr[c] + ")) return " + std::to_string(c + 1) + ";   // " + ir->knames[c] + "\n";
            }
        s += "    return 0; }\n";
    }
    s += "    default: return 0;\n    }\n}\n";
    s += kEngine;
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
    IRCK(cudaLibraryGetKernel(&ir->k_root, ir->lib, "ir_root"));
    IRCK(cudaLibraryGetKernel(&ir->k_count, ir->lib, "ir_count"));
    IRCK(cudaLibraryGetKernel(&ir->k_emit, ir->lib, "ir_emit"));
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
int scan(beast_ir *ir, const unsigned long long *cnt, unsigned long long n, unsigned long long *off,
         cudaStream_t st, unsigned long long *total) {
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
        if (launch(ir, ir->k_top, 1, 32, st, a) != BEAST_OK) return BEAST_ERR_CUDA;
    }
    {
        const unsigned g = (unsigned)std::max(1ull, (n + 255) / 256);
        void *a[] = {(void *)&off, (void *)&n, (void *)&ts, (void *)&tot};
        if (launch(ir, ir->k_add, g, 256, st, a) != BEAST_OK) return BEAST_ERR_CUDA;
    }
    IRCK(cudaMemcpyAsync(total, tot, 8, cudaMemcpyDeviceToHost, st));
    IRCK(cudaFreeAsync(ts, st));
    IRCK(cudaStreamSynchronize(st));
    return BEAST_OK;
}

int run(beast_ir *ir, cudaStream_t st, long long *out, unsigned long long capacity, unsigned long long *written,
        unsigned long long *visits, unsigned long long *rejected, bool emit_last) {
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
    IRCK(cudaMallocAsync((void **)&stats, (size_t)(NI + NC + 1) * 8, st));
    IRCK(cudaMemsetAsync(stats, 0, (size_t)(NI + NC + 1) * 8, st));
    pruned_d = (int *)(stats + NI + NC);
    {
        void *a[] = {(void *)&stats, (void *)&pruned_d};
        if (launch(ir, ir->k_root, 1, 1, st, a) != BEAST_OK) return BEAST_ERR_CUDA;
    }
    int pruned = 0;
    IRCK(cudaMemcpyAsync(&pruned, pruned_d, sizeof(int), cudaMemcpyDeviceToHost, st));
    IRCK(cudaStreamSynchronize(st));
    unsigned long long n_par = pruned ? 0 : 1;
    long long *par = nullptr;   // level -1: one empty tuple
    int rc = BEAST_OK;
    unsigned long long total = 0;
    const unsigned grid = (unsigned)ir->sm_count * 8;
    for (int k = 0; k < NI && n_par; ++k) {
        unsigned long long *cnt = nullptr, *off = nullptr;
        IRCK(cudaMallocAsync((void **)&cnt, (n_par + 1) * 8, st));
        IRCK(cudaMallocAsync((void **)&off, (n_par + 1) * 8, st));
        {
            const long long *pc = par;
            void *a[] = {(void *)&k, (void *)&pc, (void *)&n_par, (void *)&cnt, (void *)&stats};
            rc = launch(ir, ir->k_count, grid, 256, st, a);
        }
        if (rc == BEAST_OK) rc = scan(ir, cnt, n_par, off, st, &total);
        long long *child = nullptr;
        const bool last = k == NI - 1;
        if (rc == BEAST_OK && (!last || emit_last) && total) {
            if (last) {
                if (total > capacity) rc = BEAST_ERR_CAPACITY;
                else child = out;
            } else {
                const cudaError_t e = cudaMallocAsync((void **)&child, total * (unsigned long long)(k + 1) * 8, st);
                if (e != cudaSuccess) {
                    ir->err = "out of device memory for level " + std::to_string(k) + " (" + std::to_string(total) +
                              " tuples)";
                    rc = BEAST_ERR_WORKSPACE;
                }
            }
            if (rc == BEAST_OK) {
                const long long *pc = par;
                void *a[] = {(void *)&k, (void *)&pc, (void *)&n_par, (void *)&off, (void *)&child};
                rc = launch(ir, ir->k_emit, grid, 256, st, a);
            }
        }
        cudaFreeAsync(cnt, st);
        cudaFreeAsync(off, st);
        if (par) cudaFreeAsync(par, st);
        par = (last || rc != BEAST_OK) ? nullptr : child;
        n_par = total;
        if (rc != BEAST_OK) {
            if (child && child != out) cudaFreeAsync(child, st);
            break;
        }
    }
    if (NI == 0) total = pruned ? 0 : 1;
    std::vector<unsigned long long> h(NI + NC);
    if (NI + NC) IRCK(cudaMemcpyAsync(h.data(), stats, (size_t)(NI + NC) * 8, cudaMemcpyDeviceToHost, st));
    IRCK(cudaFreeAsync(stats, st));
    IRCK(cudaStreamSynchronize(st));
    if (rc != BEAST_OK && rc != BEAST_ERR_CAPACITY) return rc;
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
