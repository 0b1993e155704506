// dedup.cu -- redundant-alignment post-pass (reading R14).
//
// LASTZ stops an extension on reaching a previously-discovered alignment; that skip depends on the
// sequential order of the seeds and is infeasible in parallel, so FastZ extends every seed.  This pass
// applies the skip after the fact and order-free: a record with score >= K is redundant iff another such record
// dominates it (box containment on both axes, score at least as high, strict tie-break by seed index).
//
// Parallel form (no all-pairs scan): the candidates (score >= K) are radix-sorted by t_start (stable, so equal
// keys keep seed order); a dominator b of a satisfies a.t_end - maxlen <= b.t_start <= a.t_start, where
// maxlen = the longest candidate target span, so thread p binary-searches that window in the sorted keys and
// scans it, stopping at the first dominator.  Boxes and (score, index) are gathered once into sorted SoA so the
// scan reads 16 + 8 contiguous bytes per visited candidate.
#include <cub/device/device_radix_sort.cuh>

#include "../../include/fastz.h"
#include "internal.h"

namespace fz {

// counters: [0] = number of candidates m, [1] = max candidate target span, [2] = redundant count
__global__ void k_rd_keys(fastz_alignment* __restrict__ recs, int n, uint32_t* __restrict__ keys,
                          int* __restrict__ idx, int* __restrict__ counters) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) return;
    fastz_alignment& r = recs[s];
    const uint32_t f = r.flags & ~FASTZ_FLAG_REDUNDANT;  // idempotent: the pass recomputes the bit
    r.flags = f;
    const bool cand = (f & FASTZ_FLAG_ABOVE_K) != 0;
    keys[s] = cand ? (uint32_t)r.t_start : 0xffffffffu;  // t_start < 2^31: candidates sort before the sentinel
    idx[s] = s;
    if (cand) {
        atomicAdd(&counters[0], 1);
        atomicMax(&counters[1], (int)(r.t_end - r.t_start));
    }
}

__global__ void k_rd_gather(const fastz_alignment* __restrict__ recs, int n, const int* __restrict__ idx,
                            const int* __restrict__ counters, int4* __restrict__ box, int2* __restrict__ sc) {
    const int p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n || p >= counters[0]) return;
    const int s = idx[p];
    const fastz_alignment& r = recs[s];
    box[p] = make_int4((int)r.t_start, (int)r.t_end, (int)r.q_start, (int)r.q_end);
    sc[p] = make_int2(r.score, s);
}

__global__ void k_rd_mark(fastz_alignment* __restrict__ recs, int n, const uint32_t* __restrict__ keys,
                          const int4* __restrict__ box, const int2* __restrict__ sc, int* __restrict__ counters,
                          unsigned char* __restrict__ red) {
    const int p = blockIdx.x * blockDim.x + threadIdx.x;
    const int m = counters[0];
    if (p >= n || p >= m) return;
    const int4 a = box[p];
    const int2 as = sc[p];
    // first candidate with t_start >= a.t_end - maxlen (a candidate starting earlier ends before a.t_end)
    const long long lo_key = (long long)a.y - counters[1];
    int lo = 0, hi = m;
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if ((long long)keys[mid] < lo_key) lo = mid + 1;
        else hi = mid;
    }
    auto dominated_by = [&](int q) {
        const int4 b = box[q];
        if (b.x > a.x || a.y > b.y || b.z > a.z || a.w > b.w) return false;  // box(b) must contain box(a)
        const int2 bs = sc[q];
        if (bs.x < as.x) return false;
        const bool same_box = b.x == a.x && b.y == a.y && b.z == a.z && b.w == a.w;
        return !same_box || bs.x > as.x || bs.y < as.y;
    };
    // nearest starts first: copies of one alignment (many seeds on one homologous block) share t_start and sit
    // in seed order just before p, so a redundant copy usually stops at q = p - 1 (C5: 2.98 ms with a forward scan)
    bool dom = false;
    for (int q = p - 1; q >= lo && !dom; --q) dom = dominated_by(q);
    for (int q = p + 1; !dom && q < m && keys[q] <= (uint32_t)a.x; ++q) dom = dominated_by(q);
    if (dom) {
        red[as.y] = 1;
        recs[as.y].flags |= FASTZ_FLAG_REDUNDANT;
        atomicAdd(&counters[2], 1);
    }
}

size_t redundant_tmp_bytes(int n) {
    size_t b = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, b, (const uint32_t*)nullptr, (uint32_t*)nullptr, (const int*)nullptr,
                                    (int*)nullptr, n > 0 ? n : 1);
    return b;
}

cudaError_t launch_redundant(void* recs_, int n, void* tmp, size_t tmp_bytes, uint32_t* k1, uint32_t* k2, int* i1,
                             int* i2, int4* box, int2* sc, unsigned char* red, int* counters, cudaStream_t st) {
    cudaError_t e;
    if ((e = cudaMemsetAsync(counters, 0, 3 * sizeof(int), st)) != cudaSuccess) return e;
    if (n <= 0) return cudaSuccess;
    if ((e = cudaMemsetAsync(red, 0, (size_t)n, st)) != cudaSuccess) return e;
    auto* recs = reinterpret_cast<fastz_alignment*>(recs_);
    const int blk = 256, grid = (n + blk - 1) / blk;
    k_rd_keys<<<grid, blk, 0, st>>>(recs, n, k1, i1, counters);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    if ((e = cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, k1, k2, i1, i2, n, 0, 32, st)) != cudaSuccess) return e;
    k_rd_gather<<<grid, blk, 0, st>>>(recs, n, i2, counters, box, sc);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    k_rd_mark<<<grid, blk, 0, st>>>(recs, n, k2, box, sc, counters, red);
    return cudaGetLastError();
}

}  // namespace fz
