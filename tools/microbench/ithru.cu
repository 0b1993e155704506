// Instruction-throughput microbenchmark (sm_100a): 8 independent chains per thread, 8 warps x 8 blocks per SM.
// Prints lane-operations per clock per SM for the integer instructions the DP kernels use.
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long gt() { unsigned long long t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }

template <int K>
__global__ void kern(int iters, int* out, int s0, int s1, long long* clk) {
    int a[8], b[8], c[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) { a[k] = threadIdx.x + k; b[k] = s0 + k; c[k] = s1 * k; }
    long long c0 = clock64(); unsigned long long g0 = gt();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < 8; ++u) {
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                if (K == 0) asm volatile("max.s32 %0, %0, %1;" : "+r"(a[k]) : "r"(b[k]));                  // IMNMX
                if (K == 1) asm volatile("add.s32 %0, %0, %1;" : "+r"(a[k]) : "r"(b[k]));                  // IADD3
                if (K == 2) asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(a[k]) : "r"(b[k]), "r"(c[k])); // IMAD
                if (K == 3) a[k] = __viaddmax_s32(a[k], b[k], c[k]);                                        // VIADDMNMX
                if (K == 4) a[k] = __vimax3_s32(a[k], b[k], c[k]);                                          // VIMNMX3
                if (K == 5) asm volatile("prmt.b32 %0, %0, %1, %2;" : "+r"(a[k]) : "r"(b[k]), "r"(c[k]));   // PRMT
                if (K == 6) asm volatile("{.reg .pred p; setp.lt.s32 p, %0, %1; selp.s32 %0, %0, %2, p;}" : "+r"(a[k]) : "r"(b[k]), "r"(c[k])); // ISETP+SEL
                if (K == 7) asm volatile("{.reg .pred p; setp.lt.s32 p, %0, %1; @p mad.lo.s32 %0, %0, %2, %1;}" : "+r"(a[k]) : "r"(b[k]), "r"(c[k])); // ISETP+@IMAD
                if (K == 8) asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[k]) : "r"(b[k]), "r"(c[k]));  // LOP3
                if (K == 9) a[k] = __shfl_sync(0xffffffffu, a[k], (threadIdx.x + 31) & 31);                 // SHFL
                if (K == 10) asm volatile("min.s32 %0, %0, %1;" : "+r"(a[k]) : "r"(b[k]));                 // IMNMX (min)
                if (K == 11) { int t; asm volatile("add.s32 %0, %1, %2;" : "=r"(t) : "r"(a[k]), "r"(b[k])); asm volatile("max.s32 %0, %1, %2;" : "=r"(a[k]) : "r"(t), "r"(c[k])); } // IADD+IMNMX pair
            }
        }
    }
    long long c1 = clock64(); unsigned long long g1 = gt();
    int r = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) r ^= a[k];
    if (r == 0x12345) out[0] = r;
    if (threadIdx.x == 0 && blockIdx.x == 0) { clk[0] = c1 - c0; clk[1] = (long long)(g1 - g0); }
}

template <int K>
void run(const char* name, int sms, int opsPer) {
    int* out; long long* clk; cudaMalloc(&out, 64); cudaMalloc(&clk, 64);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    int iters = 2000;
    kern<K><<<sms * 8, 256>>>(10, out, 3, 5, clk);
    cudaEventRecord(e0);
    kern<K><<<sms * 8, 256>>>(iters, out, 3, 5, clk);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    long long c[2]; cudaMemcpy(c, clk, 16, cudaMemcpyDeviceToHost);
    double mhz = (double)c[0] / (double)c[1] * 1e3;
    double lane_ops = (double)sms * 8 * 256 * iters * 64 * opsPer;
    double per_clk_sm = lane_ops / (ms * 1e-3) / (mhz * 1e6) / sms;
    printf("%-14s %7.1f lane-instr/clk/SM  (%.2f warp-instr/clk/SMSP)  %.0f MHz  %.2f ms\n", name, per_clk_sm,
           per_clk_sm / 128.0, mhz, ms);
}

int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    run<0>("IMNMX(max)", sms, 1); run<10>("IMNMX(min)", sms, 1); run<1>("IADD", sms, 1); run<2>("IMAD", sms, 1);
    run<3>("VIADDMNMX", sms, 1); run<4>("VIMNMX3", sms, 1); run<5>("PRMT", sms, 1); run<6>("ISETP+SEL", sms, 2);
    run<7>("ISETP+@IMAD", sms, 2); run<8>("LOP3", sms, 1); run<9>("SHFL", sms, 1); run<11>("IADD+IMNMX", sms, 2);
    return 0;
}
