/*
 * ap_compute.cu — the compute-intensity workloads of PAPER.md:332-359
 * (§VI-B, Fig. 6a/6b; NEXT N4): Add, Read, Random-N, Reduce (warp shuffles),
 * FFT (warp shuffles, constant-memory twiddles) and Bitonic sort (warp
 * shuffles), each in an apointer version and a raw-pointer twin that differ
 * only in the pointer type.  "Each workload reads its data
 * using apointers and accumulates the results in a register, written back to
 * global memory at the end"; no memory tiling (one access at a
 * time through `*q; q += 32`).  4-B or 16-B loads (Fig. 6a vs 6b); a 16-B
 * load feeds four independent 32-element vectors (its x, y, z, w words).
 *
 * Layout: warp w walks units (pages) w, w+W, ... of [0, span); ADD reads its
 * second operand at the same offset + span (the region holds both vectors).
 */
#include <cuda_runtime.h>
#include <math.h>

#include "ap_internal.cuh"

#ifndef AP_BENCH_THREADS
#define AP_BENCH_THREADS 512
#endif

namespace {

__constant__ float c_tw_re[16];
__constant__ float c_tw_im[16];

struct CompArgs {
    uint64_t span;
    uint32_t unit;
    uint32_t iters; /* Random-N */
    int32_t work;
    const uint8_t* raw;
    unsigned long long* out;
};

/* --- per-lane word operations (identical in both versions) --- */
__device__ __forceinline__ uint32_t lcg_n(uint32_t x, uint32_t n) {
    for (uint32_t i = 0; i < n; ++i) x = x * 1664525u + 1013904223u;
    return x;
}

__device__ __forceinline__ uint32_t warp_sum(uint32_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

/* bitonic sort of one value per lane, ascending by lane */
__device__ __forceinline__ uint32_t warp_bitonic(uint32_t v, unsigned lane) {
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            const uint32_t o = __shfl_xor_sync(0xffffffffu, v, j);
            const bool up = ((lane & k) == 0);
            const bool lower = (lane & j) == 0;
            const uint32_t mn = o < v ? o : v, mx = o < v ? v : o;
            v = (lower == up) ? mn : mx;
        }
    }
    return v;
}

/* 32-point radix-2 DIT FFT across the warp: lane l holds x[bitrev(l)] on
 * entry (we load x[l] and permute with a shuffle), X[l] on exit. */
__device__ __forceinline__ float2 warp_fft(float2 a, unsigned lane) {
    const unsigned src = __brev(lane) >> 27;
    a.x = __shfl_sync(0xffffffffu, a.x, src);
    a.y = __shfl_sync(0xffffffffu, a.y, src);
#pragma unroll
    for (int s = 1; s <= 5; ++s) {
        const unsigned half = 1u << (s - 1);
        const float bx = __shfl_xor_sync(0xffffffffu, a.x, half);
        const float by = __shfl_xor_sync(0xffffffffu, a.y, half);
        const unsigned k = (lane & (half - 1)) * (16u >> (s - 1)); /* twiddle index */
        const float wr = c_tw_re[k], wi = c_tw_im[k];
        if (lane & half) { /* lower element: a = b_top - w * a */
            const float tr = wr * a.x - wi * a.y, ti = wr * a.y + wi * a.x;
            a.x = bx - tr;
            a.y = by - ti;
        } else { /* upper: a = a + w * b */
            const float tr = wr * bx - wi * by, ti = wr * by + wi * bx;
            a.x = a.x + tr;
            a.y = a.y + ti;
        }
    }
    return a;
}

/* one 32-bit word of input -> contribution to the lane's accumulator */
template <int WORK>
__device__ __forceinline__ unsigned long long work_word(uint32_t v, uint32_t v2, unsigned lane,
                                                        uint32_t iters) {
    if (WORK == 0) return (unsigned long long)v + v2;                     /* ADD */
    if (WORK == 1) return v;                                              /* READ */
    if (WORK == 2) return lcg_n(v, iters);                                /* RANDOM-N */
    if (WORK == 3) return warp_sum(v);                                    /* REDUCE */
    if (WORK == 4) {                                                      /* FFT */
        const float2 X = warp_fft(make_float2((float)(v & 0xffffu), (float)(v >> 16)), lane);
        const float p = X.x * X.x + X.y * X.y;
        return (unsigned long long)(p * (1.0f / 65536.0f)); /* power, scaled, truncated */
    }
    return (unsigned long long)warp_bitonic(v, lane) * (lane + 1);        /* BITONIC */
}

template <int WORK, class T>
__device__ __forceinline__ unsigned long long work_elem(const T& v, const T& v2, unsigned lane,
                                                        uint32_t iters);
template <int WORK>
__device__ __forceinline__ unsigned long long work_elem(const uint32_t& v, const uint32_t& v2,
                                                        unsigned lane, uint32_t iters) {
    return work_word<WORK>(v, v2, lane, iters);
}
template <int WORK>
__device__ __forceinline__ unsigned long long work_elem(const uint4& v, const uint4& v2,
                                                        unsigned lane, uint32_t iters) {
    return work_word<WORK>(v.x, v2.x, lane, iters) + work_word<WORK>(v.y, v2.y, lane, iters) +
           work_word<WORK>(v.z, v2.z, lane, iters) + work_word<WORK>(v.w, v2.w, lane, iters);
}

/* Per-access loops keep up to AP_COMPUTE_PIPE accesses in flight per lane:
 * access j + D is dereferenced (and its pointer moved on) before the value of
 * access j is used, so no check or fault of a later access waits for an
 * earlier access's data (the same source for both pointer types).  Built
 * for AP_COMPUTE_MINB CTAs of 512 threads per SM (1 = 128 registers: at the
 * Fig. 6 sweep's 148 thread blocks, 16 warps per SM, each with 8 reads in
 * flight). */
#ifndef AP_COMPUTE_MINB
#define AP_COMPUTE_MINB 1
#endif
#ifndef AP_COMPUTE_PIPE
#define AP_COMPUTE_PIPE 8
#endif
/* ADD keeps two values per access in the ring */
#ifndef AP_COMPUTE_PIPE_ADD
#define AP_COMPUTE_PIPE_ADD (AP_COMPUTE_PIPE > 1 ? AP_COMPUTE_PIPE / 2 : 1)
#endif

/* one access of the Fig. 6 loop through apointers: `v = *q` (and `v2 = *q2`
 * for ADD), then both pointers move on */
template <class T, int WORK>
struct ap_access {
    ap::ptr<T> q, q2;
    __device__ __forceinline__ void next(T& v, T& v2) {
        if (WORK == 0) {
            /* ADD holds two pointers: never fault one while the other pins a
             * frame of a recycled cache (R-A19); checked on the miss path */
            v = q.deref_releasing(q2);
            q += 32;
            v2 = q2.deref_releasing(q);
            q2 += 32;
        } else {
            v = *q;
            q += 32;
        }
    }
};
template <class T, int WORK>
struct raw_access {
    const T* q;
    int64_t second;
    __device__ __forceinline__ void next(T& v, T& v2) {
        v = ap::detail::ld_data<T>(q);
        if (WORK == 0) v2 = ap::detail::ld_data<T>(q + second);
        q += 32;
    }
};

template <class T, int WORK, class A>
__device__ __forceinline__ void compute_unit(A& acc_ptr, uint32_t per_unit, unsigned lane,
                                             uint32_t iters, unsigned long long& acc) {
    constexpr int D = WORK == 0 ? AP_COMPUTE_PIPE_ADD : AP_COMPUTE_PIPE;
    uint32_t j = 0;
    if (D > 1 && per_unit >= (uint32_t)D) {
        T v[D], v2[D];
#pragma unroll
        for (int d = 0; d < D; ++d) {
            v2[d] = T{};
            acc_ptr.next(v[d], v2[d]);
        }
        for (; j + 2 * D <= per_unit; j += D) {
#pragma unroll
            for (int d = 0; d < D; ++d) {
                T nv, nv2{};
                acc_ptr.next(nv, nv2);
                acc += work_elem<WORK>(v[d], v2[d], lane, iters);
                v[d] = nv;
                v2[d] = nv2;
            }
        }
#pragma unroll
        for (int d = 0; d < D; ++d) acc += work_elem<WORK>(v[d], v2[d], lane, iters);
        j += D;
    }
    for (; j < per_unit; ++j) {
        T v, v2{};
        acc_ptr.next(v, v2);
        acc += work_elem<WORK>(v, v2, lane, iters);
    }
}

template <class T, int WORK, bool APTR>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_COMPUTE_MINB)
    k_compute(const ap::dev_cache* __restrict__ c, uint32_t region, const CompArgs a) {
    constexpr uint32_t E = sizeof(T);
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const unsigned lane = threadIdx.x & 31;
    const uint64_t w = t >> 5;
    const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nunits = a.span / a.unit;
    const uint32_t per_unit = a.unit / (32 * E);
    const int64_t second = (int64_t)(a.span / E); /* ADD: b = a + span */
    unsigned long long acc = 0;
    for (uint64_t u = w; u < nunits; u += W) {
        const uint64_t e0 = u * (a.unit / E) + lane;
        if constexpr (APTR) {
            ap_access<T, WORK> p;
            p.q = ap::gvmmap<T>(c, region, e0 * E);
            if (WORK == 0) p.q2 = ap::gvmmap<T>(c, region, (e0 + second) * E);
            compute_unit<T, WORK>(p, per_unit, lane, a.iters, acc);
        } else {
            raw_access<T, WORK> p{reinterpret_cast<const T*>(a.raw) + e0, second};
            compute_unit<T, WORK>(p, per_unit, lane, a.iters, acc);
        }
    }
    a.out[t] = acc;
}

template <class T, bool APTR>
cudaError_t launch_work(const ap_cache_s* c, ap_region_t region, const ap_compute_cfg* cfg,
                        const CompArgs& a, cudaStream_t s) {
    switch (cfg->work) {
        case 0: k_compute<T, 0, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a); break;
        case 1: k_compute<T, 1, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a); break;
        case 2: k_compute<T, 2, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a); break;
        case 3: k_compute<T, 3, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a); break;
        case 4: k_compute<T, 4, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a); break;
        default: k_compute<T, 5, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
    }
    return cudaGetLastError();
}

bool g_tw_ready[64] = {};

}  // namespace

extern "C" int ap_bench_compute(ap_cache_t c, ap_region_t region, const ap_compute_cfg* cfg,
                                uint64_t* out_dev, void* stream) {
    if (!ap_region_ok(c, region) || !cfg || !out_dev) return AP_EINVAL;
    const uint32_t E = cfg->elem_bytes;
    if ((E != 4 && E != 16) || cfg->work < 0 || cfg->work > 5) return AP_EINVAL;
    if (cfg->grid == 0 || cfg->block == 0 || cfg->block > AP_BENCH_THREADS || cfg->block % 32)
        return AP_EINVAL;
    const uint64_t need = cfg->work == 0 ? 2 * cfg->span_bytes : cfg->span_bytes;
    if (cfg->span_bytes == 0 || need > c->reg[region].bytes || cfg->span_bytes % c->page)
        return AP_EINVAL;
    if (cfg->mode == AP_MODE_RAW && !cfg->raw_base) return AP_EINVAL;
    ap_device_guard g(c->device);
    if (c->device >= 0 && c->device < 64 && !g_tw_ready[c->device]) {
        float re[16], im[16];
        for (int k = 0; k < 16; ++k) { /* w^k = exp(-2*pi*i*k/32) */
            re[k] = (float)cos(-2.0 * M_PI * k / 32.0);
            im[k] = (float)sin(-2.0 * M_PI * k / 32.0);
        }
        AP_CUDA_TRY(cudaMemcpyToSymbol(c_tw_re, re, sizeof re));
        AP_CUDA_TRY(cudaMemcpyToSymbol(c_tw_im, im, sizeof im));
        g_tw_ready[c->device] = true;
    }
    CompArgs a{cfg->span_bytes, c->page, cfg->iters, cfg->work, (const uint8_t*)cfg->raw_base,
               (unsigned long long*)out_dev};
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    const bool aptr = cfg->mode == AP_MODE_APOINTER;
    if (E == 4) e = aptr ? launch_work<uint32_t, true>(c, region, cfg, a, s)
                         : launch_work<uint32_t, false>(c, region, cfg, a, s);
    else e = aptr ? launch_work<uint4, true>(c, region, cfg, a, s)
                  : launch_work<uint4, false>(c, region, cfg, a, s);
    AP_CUDA_TRY(e);
    return AP_OK;
}
