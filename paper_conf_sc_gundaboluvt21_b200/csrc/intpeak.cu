// intpeak.cu -- INT32 throughput microbenchmark for the roofline denominator.
// Eight independent dependency chains per thread of the integer ops the DP uses (IMNMX, IADD3 and the fused
// add-max VIADDMNMX), on every SM at full occupancy; reports lane-operations per second (one SASS integer
// instruction on one lane = one op) and the SM clock observed through clock64().
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>

#include "internal.h"

namespace fz {

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

template <int KIND>
__global__ void k_ipeak(int iters, int* out, int seed, long long* cycles) {
    const unsigned long long g0 = gtimer();
    int a[8], x[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        a[k] = threadIdx.x * 7 + k + seed;
        x[k] = seed * (k + 3);
    }
    const long long c0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                if (KIND == 0) asm volatile("max.s32 %0, %0, %1;" : "+r"(a[k]) : "r"(x[k] ^ u));
                else if (KIND == 1) asm volatile("add.s32 %0, %0, %1;" : "+r"(a[k]) : "r"(x[k]));
                else a[k] = __viaddmax_s32(a[k], x[k], x[(k + 1) & 7] ^ a[(k + 3) & 7]);
            }
        }
    }
    const long long c1 = clock64();
    const unsigned long long g1 = gtimer();
    int r = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) r ^= a[k];
    if (r == 0x7fffffff) out[0] = r;
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        cycles[0] = c1 - c0;
        cycles[1] = (long long)(g1 - g0);
    }
}

template <int KIND>
static cudaError_t run_kind(int sms, int iters, int* out, long long* cyc, float* ms) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int blocks = sms * 8, threads = 256;
    k_ipeak<KIND><<<blocks, threads>>>(iters / 8, out, 1, cyc);  // warm-up
    cudaEventRecord(e0);
    k_ipeak<KIND><<<blocks, threads>>>(iters, out, 1, cyc);
    cudaEventRecord(e1);
    cudaError_t e = cudaEventSynchronize(e1);
    cudaEventElapsedTime(ms, e0, e1);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t int_peak_run(int device, float target_ms, double* ops_per_s, double* mhz) {
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return e;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    int* out = nullptr;
    long long* cyc = nullptr;
    if ((e = cudaMalloc(&out, 64)) != cudaSuccess) return e;
    if ((e = cudaMalloc(&cyc, 64)) != cudaSuccess) return e;
    double best = 0, best_mhz = 0;
    const bool verbose = getenv("FASTZ_INTPEAK_VERBOSE") != nullptr;
    for (int kind = 0; kind < 3; ++kind) {
        int iters = 256;
        float ms = 0;
        for (int rep = 0; rep < 12; ++rep) {
            e = kind == 0 ? run_kind<0>(sms, iters, out, cyc, &ms)
                          : (kind == 1 ? run_kind<1>(sms, iters, out, cyc, &ms) : run_kind<2>(sms, iters, out, cyc, &ms));
            if (e != cudaSuccess) return e;
            if (ms >= target_ms) break;
            iters = (int)(iters * (ms > 0.05f ? 1.2f * target_ms / ms : 8.0f));
        }
        long long c[2] = {0, 1};
        cudaMemcpy(c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
        const double ops = (double)sms * 8 * 256 * (double)iters * 16 * 8;
        const double rate = ops / (ms * 1e-3);
        const double mhz_k = c[1] > 0 ? (double)c[0] / (double)c[1] * 1e3 : 0.0;  // cycles per ns -> MHz
        if (verbose)
            fprintf(stderr, "int_peak kind %d (%s): %.3f Tops/s, %.1f lane-ops/clk/SM at %.0f MHz\n", kind,
                    kind == 0 ? "IMNMX" : (kind == 1 ? "IADD" : "VIADDMNMX"), rate / 1e12,
                    mhz_k > 0 ? rate / (sms * mhz_k * 1e6) : 0.0, mhz_k);
        if (rate > best) {
            best = rate;
            best_mhz = mhz_k;
        }
    }
    cudaFree(out);
    cudaFree(cyc);
    *ops_per_s = best;
    *mhz = best_mhz;
    return cudaSuccess;
}

}  // namespace fz
