// Pipe-throughput microbenchmark (sm_100a): warp instructions per clock per
// SM for the integer instructions the packed scan can use.  Each thread runs
// 8 independent chains; 64 warps/SM.  Usage: ./pipes
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define REP 8192
template <int MODE>
__global__ void kern(uint32_t *out, uint32_t a, uint32_t b, long long *cyc) {
    uint32_t x[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x * (i + 3) + a;
    const uint32_t c = b ^ threadIdx.x, d = b + 7 * threadIdx.x;
    long long t0 = clock64();
    for (int r = 0; r < REP; ++r) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (MODE == 0) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[i]) : "r"(c), "r"(d));          // IMAD
            if (MODE == 1) asm volatile("add.u16x2 %0, %0, %1;" : "+r"(x[i]) : "r"(c));                       // VIADD.16x2
            if (MODE == 2) asm volatile("{.reg .b32 t; add.u32 t, %0, %1; add.u32 %0, t, %2;}" : "+r"(x[i]) : "r"(c), "r"(d));  // IADD3
            if (MODE == 3) asm volatile("{.reg .b32 t; min.u16x2 t, %0, %1; min.u16x2 %0, t, %2;}" : "+r"(x[i]) : "r"(c), "r"(d)); // VIMNMX3
            if (MODE == 4) {   // 1 IMAD + 1 VIADD16x2
                asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[i]) : "r"(c), "r"(d));
                asm volatile("add.u16x2 %0, %0, %1;" : "+r"(x[(i + 4) & 7]) : "r"(c));
            }
            if (MODE == 5) {   // 1 IMAD + 1 IADD3
                asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[i]) : "r"(c), "r"(d));
                asm volatile("{.reg .b32 t; add.u32 t, %0, %1; add.u32 %0, t, %2;}" : "+r"(x[(i + 4) & 7]) : "r"(c), "r"(d));
            }
            if (MODE == 6) {   // 1 VIADD16x2 + 1 VIMNMX3
                asm volatile("add.u16x2 %0, %0, %1;" : "+r"(x[i]) : "r"(c));
                asm volatile("{.reg .b32 t; min.u16x2 t, %0, %1; min.u16x2 %0, t, %2;}" : "+r"(x[(i + 4) & 7]) : "r"(c), "r"(d));
            }
            if (MODE == 7) {   // 1 IMAD + 1 VIMNMX3
                asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[i]) : "r"(c), "r"(d));
                asm volatile("{.reg .b32 t; min.u16x2 t, %0, %1; min.u16x2 %0, t, %2;}" : "+r"(x[(i + 4) & 7]) : "r"(c), "r"(d));
            }
            if (MODE == 8) {   // 1 IMAD + 1 VIADD16x2 + 1 VIMNMX3
                asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[i]) : "r"(c), "r"(d));
                asm volatile("add.u16x2 %0, %0, %1;" : "+r"(x[(i + 3) & 7]) : "r"(c));
                asm volatile("{.reg .b32 t; min.u16x2 t, %0, %1; min.u16x2 %0, t, %2;}" : "+r"(x[(i + 5) & 7]) : "r"(c), "r"(d));
            }
            if (MODE == 10) asm volatile("{.reg .b32 t; add.u16x2 t, %1, %2; min.u16x2 %0, %0, t;}" : "+r"(x[i]) : "r"(c ^ i), "r"(d));  // VIADDMNMX
            if (MODE == 11) {   // 2 VIADDMNMX + 1 IMAD
                asm volatile("{.reg .b32 t; add.u16x2 t, %1, %2; min.u16x2 %0, %0, t;}" : "+r"(x[i]) : "r"(c ^ i), "r"(d));
                asm volatile("{.reg .b32 t; add.u16x2 t, %1, %2; min.u16x2 %0, %0, t;}" : "+r"(x[(i + 2) & 7]) : "r"(c + i), "r"(d));
                asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[(i + 4) & 7]) : "r"(c), "r"(d));
            }
            if (MODE == 12) {   // 2 IMAD + 1 VIMNMX3 + 1 VIADDMNMX
                asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[i]) : "r"(c), "r"(d));
                asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[(i + 1) & 7]) : "r"(c), "r"(d));
                asm volatile("{.reg .b32 t; min.u16x2 t, %0, %1; min.u16x2 %0, t, %2;}" : "+r"(x[(i + 3) & 7]) : "r"(c), "r"(d));
                asm volatile("{.reg .b32 t; add.u16x2 t, %1, %2; min.u16x2 %0, %0, t;}" : "+r"(x[(i + 5) & 7]) : "r"(c ^ i), "r"(d));
            }
            if (MODE == 13) asm volatile("{.reg .b32 t; min.u16x2 %0, %0, %1;}" : "+r"(x[i]) : "r"(c ^ i));  // VIMNMX 2-input
            if (MODE == 14) {   // IADD3 + VIMNMX3
                asm volatile("{.reg .b32 t; add.u32 t, %0, %1; add.u32 %0, t, %2;}" : "+r"(x[i]) : "r"(c), "r"(d));
                asm volatile("{.reg .b32 t; min.u16x2 t, %0, %1; min.u16x2 %0, t, %2;}" : "+r"(x[(i + 4) & 7]) : "r"(c), "r"(d));
            }
            if (MODE == 9) asm volatile("{.reg .b32 t; mul.lo.u32 t, %1, 5; add.u32 %0, %0, t;}" : "+r"(x[i]) : "r"(c));  // IMAD imm
        }
    }
    long long t1 = clock64();
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) s ^= x[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int MODE>
void run(const char *name, int ipi, int sms) {
    uint32_t *o; long long *c;
    const int blocks = sms * 8, threads = 256;   // 64 warps / SM
    cudaMalloc(&o, blocks * threads * 4); cudaMalloc(&c, blocks * 8);
    kern<MODE><<<blocks, threads>>>(o, 1, 2, c);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<MODE><<<blocks, threads>>>(o, 1, 2, c);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    long long h[4]; cudaMemcpy(h, c, sizeof(h), cudaMemcpyDeviceToHost);
    double warp_inst = (double)blocks * (threads / 32) * REP * 8 * ipi;
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    double cycles = ms * 1e-3 * clk * 1e3;
    printf("%-28s %6.3f warp-inst/clk/SM (%.3f ms, blk0 %lld cyc)\n", name, warp_inst / cycles / sms, ms, h[0]);
    cudaFree(o); cudaFree(c);
}

int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    run<0>("IMAD", 1, sms);
    run<1>("VIADD.16x2", 1, sms);
    run<2>("IADD3", 1, sms);
    run<3>("VIMNMX3.U16x2", 1, sms);
    run<4>("IMAD+VIADD.16x2", 2, sms);
    run<5>("IMAD+IADD3", 2, sms);
    run<6>("VIADD.16x2+VIMNMX3", 2, sms);
    run<7>("IMAD+VIMNMX3", 2, sms);
    run<8>("IMAD+VIADD.16x2+VIMNMX3", 3, sms);
    run<9>("IMAD(imm)", 1, sms);
    run<10>("VIADDMNMX.U16x2", 1, sms);
    run<11>("2 VIADDMNMX + IMAD", 3, sms);
    run<12>("2 IMAD+VIMNMX3+VIADDMNMX", 4, sms);
    run<13>("VIMNMX.U16x2", 1, sms);
    run<14>("IADD3+VIMNMX3", 2, sms);
    return 0;
}
