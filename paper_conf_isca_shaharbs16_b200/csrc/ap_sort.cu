/*
 * ap_sort.cu — the library's own stable radix sort of (key, value) pairs,
 * used inside the timed collage step (the locality schedules order blocks /
 * units by their LSH keys) and by the bucket-index build
 * ("images are placed in buckets indexed by the LSH keys").
 *
 * LSD over 8-bit digits of the low `bits` bits of the key.  One pass:
 *   1. k_sort_hist: each CTA counts the digits of its tile (2048 keys) into
 *      shared memory and writes them digit-major, counts[d][cta];
 *   2. k_sort_scan: one CTA turns counts into exclusive offsets (digit-major
 *      order = all smaller digits first, then the same digit of earlier
 *      CTAs: the stable global position of each (digit, CTA) run);
 *   3. k_sort_scatter: each warp of a CTA owns 256 consecutive keys of the
 *      tile; per-warp digit counts are prefixed over the warps, then every
 *      warp walks its keys 32 at a time in order, ranks equal digits with
 *      __match_any_sync (rank = earlier lanes of the same digit) and writes
 *      key and value to their final position.  Order of equal keys is kept.
 */
#include <cuda_runtime.h>

#include "ap_internal.cuh"

namespace {

constexpr int SORT_THREADS = 256;
constexpr int SORT_WARPS = SORT_THREADS / 32;
constexpr int SORT_PER_WARP = 256;
constexpr uint64_t SORT_TILE = (uint64_t)SORT_WARPS * SORT_PER_WARP;

template <class K>
__global__ void __launch_bounds__(SORT_THREADS) k_sort_hist(const K* __restrict__ keys, uint64_t n,
                                                             int shift, uint32_t* counts) {
    __shared__ uint32_t h[256];
    h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t t0 = blockIdx.x * SORT_TILE;
    for (uint64_t i = threadIdx.x; i < SORT_TILE && t0 + i < n; i += SORT_THREADS)
        atomicAdd(&h[(uint32_t)(keys[t0 + i] >> shift) & 255u], 1u);
    __syncthreads();
    counts[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x] = h[threadIdx.x];
}

/* exclusive scan of counts[0 .. total) in place, one CTA of 1024 threads,
 * each thread a contiguous chunk */
__global__ void __launch_bounds__(1024) k_sort_scan(uint32_t* counts, uint64_t total) {
    __shared__ uint32_t part[1024];
    const uint64_t per = (total + 1023) / 1024;
    const uint64_t b = threadIdx.x * per, e = b + per < total ? b + per : total;
    uint32_t s = 0;
    for (uint64_t i = b; i < e; ++i) s += counts[i];
    part[threadIdx.x] = s;
    __syncthreads();
    for (int o = 1; o < 1024; o <<= 1) { /* Hillis-Steele inclusive scan */
        const uint32_t v = threadIdx.x >= (unsigned)o ? part[threadIdx.x - o] : 0u;
        __syncthreads();
        part[threadIdx.x] += v;
        __syncthreads();
    }
    uint32_t run = threadIdx.x ? part[threadIdx.x - 1] : 0u;
    for (uint64_t i = b; i < e; ++i) {
        const uint32_t c = counts[i];
        counts[i] = run;
        run += c;
    }
}

template <class K>
__global__ void __launch_bounds__(SORT_THREADS)
    k_sort_scatter(const K* __restrict__ kin, const uint32_t* __restrict__ vin, K* __restrict__ kout,
                   uint32_t* __restrict__ vout, uint64_t n, int shift,
                   const uint32_t* __restrict__ offs) {
    __shared__ uint32_t wcnt[SORT_WARPS][256];
    const unsigned tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    for (unsigned i = tid; i < SORT_WARPS * 256; i += SORT_THREADS) (&wcnt[0][0])[i] = 0;
    __syncthreads();
    const uint64_t sub = blockIdx.x * SORT_TILE + (uint64_t)warp * SORT_PER_WARP;
    unsigned lt;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
    /* 1. this warp's digit counts */
    for (int it = 0; it < SORT_PER_WARP / 32; ++it) {
        const uint64_t i = sub + it * 32 + lane;
        const uint32_t d = i < n ? ((uint32_t)(kin[i] >> shift) & 255u) : 256u;
        const unsigned grp = __match_any_sync(0xffffffffu, d);
        if (d < 256u && (grp & lt) == 0) wcnt[warp][d] += __popc(grp);
        __syncwarp();
    }
    __syncthreads();
    /* 2. global start of each (digit, warp) run */
    {
        const unsigned d = tid; /* SORT_THREADS == 256 digits */
        uint32_t run = offs[(uint64_t)d * gridDim.x + blockIdx.x];
        for (int w = 0; w < SORT_WARPS; ++w) {
            const uint32_t c = wcnt[w][d];
            wcnt[w][d] = run;
            run += c;
        }
    }
    __syncthreads();
    /* 3. scatter in order */
    for (int it = 0; it < SORT_PER_WARP / 32; ++it) {
        const uint64_t i = sub + it * 32 + lane;
        const bool ok = i < n;
        const K k = ok ? kin[i] : K(0);
        const uint32_t d = ok ? ((uint32_t)(k >> shift) & 255u) : 256u;
        const unsigned grp = __match_any_sync(0xffffffffu, d);
        uint32_t pos = 0;
        if (ok) pos = wcnt[warp][d] + __popc(grp & lt);
        __syncwarp();
        if (ok) {
            kout[pos] = k;
            vout[pos] = vin[i];
            if ((grp & lt) == 0) wcnt[warp][d] += __popc(grp);
        }
        __syncwarp();
    }
}

}  // namespace

size_t ap_sort_scratch_bytes(uint64_t n) {
    const uint64_t tiles = (n + SORT_TILE - 1) / SORT_TILE;
    return (size_t)(256 * (tiles ? tiles : 1) * 4);
}

template <class K>
int ap_sort_pairs(K* keys, K* keys_alt, uint32_t* vals, uint32_t* vals_alt, uint64_t n, int bits,
                  void* scratch, cudaStream_t s, bool* in_alt) {
    *in_alt = false;
    if (n == 0) return AP_OK;
    if (n > 0xffffffffull || bits < 0 || bits > (int)(8 * sizeof(K))) return AP_EINVAL;
    const uint64_t tiles = (n + SORT_TILE - 1) / SORT_TILE;
    if (tiles > 0x7fffffffull) return AP_ERANGE;
    uint32_t* counts = (uint32_t*)scratch;
    K* ki = keys;
    K* ko = keys_alt;
    uint32_t* vi = vals;
    uint32_t* vo = vals_alt;
    for (int shift = 0; shift < bits; shift += 8) {
        k_sort_hist<K><<<(unsigned)tiles, SORT_THREADS, 0, s>>>(ki, n, shift, counts);
        k_sort_scan<<<1, 1024, 0, s>>>(counts, 256 * tiles);
        k_sort_scatter<K><<<(unsigned)tiles, SORT_THREADS, 0, s>>>(ki, vi, ko, vo, n, shift, counts);
        K* tk = ki;
        ki = ko;
        ko = tk;
        uint32_t* tv = vi;
        vi = vo;
        vo = tv;
        *in_alt = !*in_alt;
    }
    AP_CUDA_TRY(cudaGetLastError());
    return AP_OK;
}

template int ap_sort_pairs<unsigned long long>(unsigned long long*, unsigned long long*, uint32_t*,
                                               uint32_t*, uint64_t, int, void*, cudaStream_t,
                                               bool*);
template int ap_sort_pairs<uint32_t>(uint32_t*, uint32_t*, uint32_t*, uint32_t*, uint64_t, int,
                                     void*, cudaStream_t, bool*);
