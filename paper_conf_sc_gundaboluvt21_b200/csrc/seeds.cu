// seeds.cu -- seeding + ungapped filter on the GPU, the stage before the gapped
// extension: "a lightweight exact-match search identifies short sequences (19 base pairs long)
// to serve as seed sites ... the second stage filters the seed sites to obtain a shorter list of promising seed
// sites ... the third stage extends the filtered seed sites".  Semantics = readings S1-S6 (spaced
// 12of19 seed with one transition, ungapped x-drop, HSP threshold, midpoint anchor -- LASTZ defaults [ext]).
//
// Pipeline (all on the context's stream):
//   k_seed_keys     spaced-seed word of every target position (2 bits per care position) -> (word, position)
//   radix sort      CUB, stable: positions ascending inside a word
//   k_bucket_start  dense bucket starts for w <= 12 care positions (4^w + 1 ints); binary search otherwise
//   per query chunk (sized so the chunk's hits fit the hit buffer):
//     k_seed_count  hits per query position (exact word + one transition per care position)
//     scan          CUB exclusive sum -> hit offsets (one D2H of the chunk total)
//     k_seed_write  (t, q) hits
//     k_ungapped    one thread per hit: x-drop walk right and left along the diagonal over the 2-bit packed
//                   sequences (one 32-bit load per 16 bases), HSP + score; survivors (>= hspthresh) flagged
//     select        CUB DeviceSelect -> appended to the HSP list
//   k_hsp_keys + 2 radix sorts (LSD: (t_start, length) then (anchor t, anchor q)), k_hsp_unique + scan,
//   k_hsp_emit      deduplicated HSPs (S5) in anchor order (S6) + their anchors as fastz_seed cut points.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>

#include <algorithm>

#include "internal.h"

namespace fz {

// S1: spaced-seed word at position p: the codes at the care offsets, first care position in the highest bits
__device__ __forceinline__ uint32_t seed_word(const uint32_t* __restrict__ pk, long long p, const SeedPattern& sp) {
    const long long w0 = p >> 4;
    const int sh = (int)(p & 15);
    const unsigned long long lo = (unsigned long long)__ldg(pk + w0) | ((unsigned long long)__ldg(pk + w0 + 1) << 32);
    const uint32_t hi = __ldg(pk + w0 + 2);  // span <= 32: offsets up to sh + 31 <= 46 (buffers carry 4 pad words)
    uint32_t k = 0;
#pragma unroll 4
    for (int c = 0; c < sp.w; ++c) {
        const int o = sh + sp.off[c];
        const uint32_t b = o < 32 ? (uint32_t)(lo >> (2 * o)) & 3u : (hi >> (2 * (o - 32))) & 3u;
        k = (k << 2) | b;
    }
    return k;
}

// S7: does the word at position p have an N at a care position?  (nm == nullptr: the sequence has no N)
__device__ __forceinline__ bool care_has_n(const uint16_t* __restrict__ nm, long long p, const SeedPattern& sp) {
    if (nm == nullptr) return false;
    const long long w0 = p >> 4;
    const unsigned long long bits = (unsigned long long)__ldg(nm + w0) | ((unsigned long long)__ldg(nm + w0 + 1) << 16) |
                                    ((unsigned long long)__ldg(nm + w0 + 2) << 32);  // masks carry 4 pad words
    return ((bits >> (p & 15)) & sp.caremask) != 0;
}

__global__ void k_seed_keys(const uint32_t* __restrict__ Tf, const uint16_t* __restrict__ TfN, long long nt,
                            SeedPattern sp, uint32_t* keys, int* pos, unsigned char* valid) {
    const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= nt) return;
    keys[p] = seed_word(Tf, p, sp);
    pos[p] = (int)p;
    if (valid) valid[p] = care_has_n(TfN, p, sp) ? 0 : 1;
}

// dense bucket starts: start[k] = first sorted index with key >= k, k in [0, 4^w]
__global__ void k_bucket_start(const uint32_t* __restrict__ skeys, long long nt, int* start, long long nkeys) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nt) return;
    const long long k = skeys[i];
    const long long prev = i ? (long long)skeys[i - 1] : -1;
    for (long long kk = prev + 1; kk <= k; ++kk) start[kk] = (int)i;
    if (i == nt - 1)
        for (long long kk = k + 1; kk <= nkeys; ++kk) start[kk] = (int)nt;
}

struct SeedIndex {
    const uint32_t* skeys;  // sorted words
    const int* spos;        // target positions in word order
    const int* start;       // dense bucket starts (nullptr: binary search)
    long long nt;
};

__device__ __forceinline__ void bucket(const SeedIndex& ix, uint32_t k, long long& lo, long long& hi) {
    if (ix.start) {
        lo = ix.start[k];
        hi = ix.start[k + 1];
        return;
    }
    long long a = 0, b = ix.nt;
    while (a < b) {
        const long long m = (a + b) >> 1;
        if (ix.skeys[m] < k) a = m + 1; else b = m;
    }
    lo = a;
    b = ix.nt;
    while (a < b) {
        const long long m = (a + b) >> 1;
        if (ix.skeys[m] <= k) a = m + 1; else b = m;
    }
    hi = a;
}

// S2: variant 0 = the exact word; variant 1 + c = a transition (A<->G, C<->T: code xor 2) at care position c
__device__ __forceinline__ uint32_t variant(uint32_t k0, int v, int w) {
    return v == 0 ? k0 : k0 ^ (2u << (2 * (w - v)));
}

__global__ void k_seed_count(const uint32_t* __restrict__ Qf, const uint16_t* __restrict__ QfN, long long q0,
                             long long nq, SeedPattern sp, int nvar, SeedIndex ix, long long* cnt) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i > nq) return;
    if (i == nq || care_has_n(QfN, q0 + i, sp)) {  // S7
        cnt[i] = 0;
        return;
    }
    const uint32_t k0 = seed_word(Qf, q0 + i, sp);
    long long n = 0;
    for (int v = 0; v < nvar; ++v) {
        long long lo, hi;
        bucket(ix, variant(k0, v, sp.w), lo, hi);
        n += hi - lo;
    }
    cnt[i] = n;
}

__global__ void k_seed_write(const uint32_t* __restrict__ Qf, const uint16_t* __restrict__ QfN, long long q0,
                             long long nq, SeedPattern sp, int nvar, SeedIndex ix, const long long* __restrict__ off,
                             int2* hits) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nq || care_has_n(QfN, q0 + i, sp)) return;  // S7
    const uint32_t k0 = seed_word(Qf, q0 + i, sp);
    long long o = off[i];
    for (int v = 0; v < nvar; ++v) {
        long long lo, hi;
        bucket(ix, variant(k0, v, sp.w), lo, hi);
        for (long long e = lo; e < hi; ++e) hits[o++] = make_int2(ix.spos[e], (int)(q0 + i));
    }
}

// Reads consecutive bases of a 2-bit packed sequence (either direction) with one load per 16 bases; with an N
// mask (nm != nullptr) an N reads as code 4.
struct BaseStream {
    const uint32_t* pk;
    const uint16_t* nm;
    long long word;
    uint32_t cur, curn;
    __device__ __forceinline__ void init(const uint32_t* p, const uint16_t* m, long long pos) {
        pk = p;
        nm = m;
        word = pos >> 4;
        cur = __ldg(pk + word);
        curn = nm ? __ldg(nm + word) : 0u;
    }
    __device__ __forceinline__ int get(long long pos) {
        const long long w = pos >> 4;
        if (w != word) {
            word = w;
            cur = __ldg(pk + w);
            curn = nm ? __ldg(nm + w) : 0u;
        }
        const int sh = (int)(pos & 15);
        return (int)((cur >> (sh * 2)) & 3u) | (int)(((curn >> sh) & 1u) << 2);
    }
};

// S3 + S4: one thread per hit.  out[h] = {t_start, q_start, length, score}; keep[h] = score >= thresh.
__global__ void k_ungapped(const int2* __restrict__ hits, long long nh, const uint32_t* __restrict__ Tf,
                           const uint32_t* __restrict__ Qf, const uint16_t* __restrict__ TfN,
                           const uint16_t* __restrict__ QfN, int tlen, int qlen, UngappedParams up, int4* out,
                           unsigned char* keep) {
    __shared__ int sub[25];
    if (threadIdx.x < 25) sub[threadIdx.x] = up.sub[threadIdx.x];
    __syncthreads();
    const long long h = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (h >= nh) return;
    const int2 hq = hits[h];
    const int t = hq.x, q = hq.y;
    BaseStream ts, qs;
    // right: (t + d, q + d), d = 0, 1, ...
    int s = 0, best_r = 0, r = 0;
    const int nr = min(tlen - t, qlen - q);
    if (nr > 0) {
        ts.init(Tf, TfN, t);
        qs.init(Qf, QfN, q);
        for (int d = 0; d < nr; ++d) {
            s += sub[5 * ts.get(t + d) + qs.get(q + d)];
            if (s > best_r) {
                best_r = s;
                r = d + 1;
            }
            if (s < best_r - up.xdrop) break;
        }
    }
    // left: (t - d, q - d), d = 1, 2, ...
    int best_l = 0, l = 0;
    s = 0;
    const int nl = min(t, q);
    if (nl > 0) {
        ts.init(Tf, TfN, t - 1);
        qs.init(Qf, QfN, q - 1);
        for (int d = 1; d <= nl; ++d) {
            s += sub[5 * ts.get(t - d) + qs.get(q - d)];
            if (s > best_l) {
                best_l = s;
                l = d;
            }
            if (s < best_l - up.xdrop) break;
        }
    }
    const int score = best_l + best_r;
    out[h] = make_int4(t - l, q - l, l + r, score);
    keep[h] = score >= up.hspthresh ? 1 : 0;
}

// sort keys of the HSP list: primary (anchor t, anchor q), secondary (t_start, length) -- S6
__global__ void k_hsp_keys(const int4* __restrict__ hs, long long n, unsigned long long* kpri,
                           unsigned long long* ksec, int* idx) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int4 h = hs[i];
    kpri[i] = ((unsigned long long)(unsigned)(h.x + h.z / 2) << 32) | (unsigned)(h.y + h.z / 2);
    ksec[i] = ((unsigned long long)(unsigned)h.x << 32) | (unsigned)h.z;
    idx[i] = (int)i;
}

__global__ void k_gather_u64(const unsigned long long* __restrict__ src, const int* __restrict__ idx, long long n,
                             unsigned long long* dst) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) dst[i] = src[idx[i]];
}

// S5: first of each run of identical HSPs (identical records are adjacent in anchor order)
__global__ void k_hsp_unique(const int4* __restrict__ hs, const int* __restrict__ order, long long n, int* flag) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i > n) return;
    if (i == n) {
        flag[i] = 0;
        return;
    }
    const int4 a = hs[order[i]];
    bool first = true;
    if (i > 0) {
        const int4 b = hs[order[i - 1]];
        first = !(a.x == b.x && a.y == b.y && a.z == b.z);
    }
    flag[i] = first ? 1 : 0;
}

__global__ void k_hsp_emit(const int4* __restrict__ hs, const int* __restrict__ order, const int* __restrict__ flag,
                           const int* __restrict__ pos, long long n, HspOut* out, long long* anchors) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n || !flag[i]) return;
    const int4 h = hs[order[i]];
    const long long o = pos[i];
    out[o].t_start = h.x;
    out[o].q_start = h.y;
    out[o].length = h.z;
    out[o].score = h.w;
    anchors[2 * o] = h.x + h.z / 2;  // S6: midpoint cut point
    anchors[2 * o + 1] = h.y + h.z / 2;
}

static inline unsigned nblk(long long n, int t = 256) { return (unsigned)((n + t - 1) / t); }

// ------------------------------------------------------------------------------------------------ launchers
cudaError_t seed_keys(const uint32_t* Tf, const uint16_t* TfN, long long nt, const SeedPattern& sp, uint32_t* keys,
                      int* pos, unsigned char* valid, cudaStream_t st) {
    if (nt <= 0) return cudaSuccess;
    k_seed_keys<<<nblk(nt), 256, 0, st>>>(Tf, TfN, nt, sp, keys, pos, valid);
    return cudaGetLastError();
}

// S7: drop target words with an N at a care position before the sort (two selects: words, positions)
cudaError_t seed_compact(void* tmp, size_t tmp_bytes, const uint32_t* kin, const int* pin, const unsigned char* valid,
                         long long nt, uint32_t* kout, int* pout, int* nsel, cudaStream_t st) {
    cudaError_t e = cub::DeviceSelect::Flagged(tmp, tmp_bytes, kin, valid, kout, nsel, (int)nt, st);
    if (e != cudaSuccess) return e;
    return cub::DeviceSelect::Flagged(tmp, tmp_bytes, pin, valid, pout, nsel, (int)nt, st);
}

size_t seed_sort_tmp_bytes(long long n) {
    size_t a = 0, b = 0, c = 0, d = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, a, (const uint32_t*)nullptr, (uint32_t*)nullptr, (const int*)nullptr,
                                    (int*)nullptr, (int)(n > 0 ? n : 1));
    cub::DeviceRadixSort::SortPairs(nullptr, b, (const unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                    (const int*)nullptr, (int*)nullptr, (int)(n > 0 ? n : 1));
    cub::DeviceScan::ExclusiveSum(nullptr, c, (const long long*)nullptr, (long long*)nullptr, (int)(n > 0 ? n + 1 : 2));
    cub::DeviceSelect::Flagged(nullptr, d, (const int4*)nullptr, (const unsigned char*)nullptr, (int4*)nullptr,
                               (int*)nullptr, (int)(n > 0 ? n : 1));
    size_t e = 0, f = 0, g = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, e, (const int*)nullptr, (int*)nullptr, (int)(n > 0 ? n + 1 : 2));
    cub::DeviceSelect::Flagged(nullptr, f, (const uint32_t*)nullptr, (const unsigned char*)nullptr, (uint32_t*)nullptr,
                               (int*)nullptr, (int)(n > 0 ? n : 1));
    cub::DeviceSelect::Flagged(nullptr, g, (const int*)nullptr, (const unsigned char*)nullptr, (int*)nullptr,
                               (int*)nullptr, (int)(n > 0 ? n : 1));
    return std::max(std::max(std::max(a, b), std::max(c, d)), std::max(e, std::max(f, g)));
}

cudaError_t seed_sort_words(void* tmp, size_t tmp_bytes, const uint32_t* kin, uint32_t* kout, const int* vin,
                            int* vout, long long n, int bits, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    return cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, kin, kout, vin, vout, (int)n, 0, bits, st);
}

cudaError_t seed_bucket_start(const uint32_t* skeys, long long nt, int* start, long long nkeys, cudaStream_t st) {
    cudaError_t e = cudaMemsetAsync(start, 0, sizeof(int) * (size_t)(nkeys + 1), st);
    if (e != cudaSuccess || nt <= 0) return e;
    k_bucket_start<<<nblk(nt), 256, 0, st>>>(skeys, nt, start, nkeys);
    return cudaGetLastError();
}

cudaError_t seed_count(const uint32_t* Qf, const uint16_t* QfN, long long q0, long long nq, const SeedPattern& sp,
                       int nvar, const uint32_t* skeys, const int* spos, const int* start, long long nt, long long* cnt,
                       long long* off, void* tmp, size_t tmp_bytes, cudaStream_t st) {
    SeedIndex ix{skeys, spos, start, nt};
    k_seed_count<<<nblk(nq + 1), 256, 0, st>>>(Qf, QfN, q0, nq, sp, nvar, ix, cnt);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    return cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, cnt, off, (int)(nq + 1), st);
}

cudaError_t seed_write_extend(const uint32_t* Tf, const uint32_t* Qf, const uint16_t* TfN, const uint16_t* QfN, int tlen,
                              int qlen, long long q0, long long nq,
                              const SeedPattern& sp, int nvar, const uint32_t* skeys, const int* spos,
                              const int* start, long long nt, const long long* off, long long nh, int2* hits,
                              const UngappedParams& up, int4* hsp, unsigned char* keep, cudaStream_t st) {
    if (nq <= 0 || nh <= 0) return cudaSuccess;
    SeedIndex ix{skeys, spos, start, nt};
    k_seed_write<<<nblk(nq), 256, 0, st>>>(Qf, QfN, q0, nq, sp, nvar, ix, off, hits);
    k_ungapped<<<nblk(nh), 256, 0, st>>>(hits, nh, Tf, Qf, TfN, QfN, tlen, qlen, up, hsp, keep);
    return cudaGetLastError();
}

cudaError_t seed_select(void* tmp, size_t tmp_bytes, const int4* hsp, const unsigned char* keep, long long nh,
                        int4* out, int* nsel, cudaStream_t st) {
    return cub::DeviceSelect::Flagged(tmp, tmp_bytes, hsp, keep, out, nsel, (int)nh, st);
}

cudaError_t seed_finish_sort(void* tmp, size_t tmp_bytes, const int4* hs, long long n, unsigned long long* k1,
                             unsigned long long* k2, int* i1, int* i2, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    k_hsp_keys<<<nblk(n), 256, 0, st>>>(hs, n, k1, k2, i1);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    // LSD: secondary key first (stable), then the primary key of the reordered records
    if ((e = cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, k2, k2 + n, i1, i2, (int)n, 0, 64, st)) != cudaSuccess)
        return e;
    k_gather_u64<<<nblk(n), 256, 0, st>>>(k1, i2, n, k2);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    return cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, k2, k1, i2, i1, (int)n, 0, 64, st);  // order -> i1
}

cudaError_t seed_unique_emit(void* tmp, size_t tmp_bytes, const int4* hs, const int* order, long long n, int* flag,
                             int* pos, HspOut* out, long long* anchors, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    k_hsp_unique<<<nblk(n + 1), 256, 0, st>>>(hs, order, n, flag);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    if ((e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, flag, pos, (int)(n + 1), st)) != cudaSuccess) return e;
    k_hsp_emit<<<nblk(n), 256, 0, st>>>(hs, order, flag, pos, n, out, anchors);
    return cudaGetLastError();
}

}  // namespace fz
