// Packed-scan loop-body microbenchmark (sm_100a): points per clock per SM of
// candidate 16-pair block bodies.  Usage: ./scan
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t body_A(uint32_t acc, uint32_t Cb, uint32_t Sp) {   // 16 IMAD + 8 VIMNMX3
    asm volatile(
        "{\n\t.reg .b32 t<16>;\n\t"
        "mad.lo.u32 t0, %2, 1, %1;\n\t mad.lo.u32 t1, %2, 2, %1;\n\t min.u16x2 %0, %0, t0;\n\t min.u16x2 %0, %0, t1;\n\t"
        "mad.lo.u32 t2, %2, 3, %1;\n\t mad.lo.u32 t3, %2, 4, %1;\n\t min.u16x2 %0, %0, t2;\n\t min.u16x2 %0, %0, t3;\n\t"
        "mad.lo.u32 t4, %2, 5, %1;\n\t mad.lo.u32 t5, %2, 6, %1;\n\t min.u16x2 %0, %0, t4;\n\t min.u16x2 %0, %0, t5;\n\t"
        "mad.lo.u32 t6, %2, 7, %1;\n\t mad.lo.u32 t7, %2, 8, %1;\n\t min.u16x2 %0, %0, t6;\n\t min.u16x2 %0, %0, t7;\n\t"
        "mad.lo.u32 t8, %2, 9, %1;\n\t mad.lo.u32 t9, %2, 10, %1;\n\t min.u16x2 %0, %0, t8;\n\t min.u16x2 %0, %0, t9;\n\t"
        "mad.lo.u32 t10, %2, 11, %1;\n\t mad.lo.u32 t11, %2, 12, %1;\n\t min.u16x2 %0, %0, t10;\n\t min.u16x2 %0, %0, t11;\n\t"
        "mad.lo.u32 t12, %2, 13, %1;\n\t mad.lo.u32 t13, %2, 14, %1;\n\t min.u16x2 %0, %0, t12;\n\t min.u16x2 %0, %0, t13;\n\t"
        "mad.lo.u32 t14, %2, 15, %1;\n\t mad.lo.u32 t15, %2, 16, %1;\n\t min.u16x2 %0, %0, t14;\n\t min.u16x2 %0, %0, t15;\n\t"
        "}" : "+r"(acc) : "r"(Cb), "r"(Sp));
    return acc;
}
// NI products by IMAD (paired into VIMNMX3), the remaining 16-NI by VIADDMNMX with invariants M[]
template <int NI>
__device__ __forceinline__ uint32_t body_mix(uint32_t acc, uint32_t Cb, uint32_t Sp, const uint32_t *M) {
#pragma unroll
    for (int j = 1; j <= NI; j += 2) {
        uint32_t a, b;
        a = Sp * (uint32_t)j + Cb;
        b = Sp * (uint32_t)(j + 1) + Cb;
        asm volatile("{.reg .b32 t; min.u16x2 t, %0, %1; min.u16x2 %0, t, %2;}" : "+r"(acc) : "r"(a), "r"(b));
    }
#pragma unroll
    for (int j = NI + 1; j <= 16; ++j)
        asm volatile("{.reg .b32 t; add.u16x2 t, %1, %2; min.u16x2 %0, %0, t;}" : "+r"(acc) : "r"(Cb), "r"(M[j - NI - 1]));
    return acc;
}

template <int V>
__global__ void __launch_bounds__(256) kern(uint32_t *out, uint32_t nb, uint32_t T) {
    const uint32_t s1 = 1 + (threadIdx.x & 63), s2 = s1 + 1 + (blockIdx.x & 7);
    const uint32_t Sp = s1 | (s2 << 16);
    uint32_t Cb = (0x10000u - T) * 0x10001u;
    const uint32_t step = Sp << 4;
    uint32_t M[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) M[j] = Sp * (uint32_t)(17 - 16 + j + (V > 0 ? V : 0));
    uint32_t acc = 0xffffffffu;
    for (uint32_t b = 0; b < nb; ++b) {
        if (V == 0) acc = body_A(acc, Cb, Sp);
        if (V == 8) acc = body_mix<8>(acc, Cb, Sp, M);
        if (V == 10) acc = body_mix<10>(acc, Cb, Sp, M);
        if (V == 12) acc = body_mix<12>(acc, Cb, Sp, M);
        if (V == 6) acc = body_mix<6>(acc, Cb, Sp, M);
        if (V == 2) acc = body_mix<2>(acc, Cb, Sp, M);
        Cb += step;
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int V>
void run(const char *name, int sms, int per_sm) {
    uint32_t *o;
    const int blocks = sms * per_sm, threads = 256, nb = 4096;
    cudaMalloc(&o, blocks * threads * 4);
    kern<V><<<blocks, threads>>>(o, nb, 777);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<V><<<blocks, threads>>>(o, nb, 777);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const double pts = (double)blocks * threads * nb * 32;
    printf("%-22s %2d warps/SM: %7.2f points/clk/SM  %.3e points/s  (%.3f ms)\n", name, per_sm * 8,
           pts / (ms * 1e-3 * clk * 1e3) / sms, pts / (ms * 1e-3), ms);
    cudaFree(o);
}

int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int per : {4, 6, 8}) {
        run<0>("A: 16 IMAD + 8 VIMNMX3", sms, per);
        run<12>("12 IMAD + 4 VIADDMNMX", sms, per);
        run<10>("10 IMAD + 6 VIADDMNMX", sms, per);
        run<8>("8 IMAD + 8 VIADDMNMX", sms, per);
        run<6>("6 IMAD + 10 VIADDMNMX", sms, per);
        run<2>("2 IMAD + 14 VIADDMNMX", sms, per);
    }
    return 0;
}
