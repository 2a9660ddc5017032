/*
 * ap_bench.cu — the apointer microbenchmarks (§VI-A/C) on
 * B200, each in two versions that differ only in the pointer type
 * ("We develop two versions of every benchmark"):
 *
 *   SEQ        warp w sweeps units w, w+W, ... of the file; lanes read
 *              consecutive elements (coalesced), `q += 32` between reads
 *              (the copy/throughput kernel, and the page
 *              walk of PAPER.md:367 "each warp accesses ... different pages in
 *              a loop, with all threads in a warp accessing the same page").
 *   UNIFORM    uniform-random element offsets, reached by pointer arithmetic
 *              from the previous offset (C2).
 *   DIVERGENT  the 32 lanes of a warp on 32 distinct pages (C3).
 *
 * Output: per-thread FNV-1a-64 over the values read (or the bytes themselves
 * for SEQ out_copy).  Workload definitions: DESIGN.md "Workloads".
 */
#include <cuda_runtime.h>

#include <algorithm>

#include "ap_internal.cuh"

/* The apointer kernels need ~120 registers once the fault path is linked
 * in; 512 threads x 128 registers = one CTA of 16 warps per SM. */
#ifndef AP_BENCH_THREADS
#define AP_BENCH_THREADS 512
#endif
#ifndef AP_BENCH_MINB
#define AP_BENCH_MINB 1
#endif
#ifndef AP_SEQ_MINB
#define AP_SEQ_MINB AP_BENCH_MINB
#endif

namespace {

constexpr uint64_t FNV_BASIS = 0xcbf29ce484222325ull;
constexpr uint64_t FNV_PRIME = 0x100000001b3ull;

__device__ __forceinline__ uint64_t fnv(uint64_t h, uint32_t v) {
    return (h ^ (uint64_t)v) * FNV_PRIME;
}
__device__ __forceinline__ uint64_t fnv(uint64_t h, unsigned long long v) {
    return (h ^ (uint64_t)v) * FNV_PRIME;
}
__device__ __forceinline__ uint64_t fnv(uint64_t h, uint4 v) {
    h = (h ^ (((uint64_t)v.y << 32) | v.x)) * FNV_PRIME;
    return (h ^ (((uint64_t)v.w << 32) | v.z)) * FNV_PRIME;
}

struct BenchArgs {
    uint64_t bytes;     /* region bytes                                 */
    uint64_t span;      /* SEQ sweep bytes                              */
    uint32_t unit;      /* SEQ unit bytes                               */
    uint32_t passes;    /* SEQ                                          */
    uint32_t reads;     /* UNIFORM / DIVERGENT                          */
    uint32_t page;      /* DIVERGENT pattern page size                  */
    uint64_t seed;
    const uint8_t* raw; /* RAW twin base                                */
    uint8_t* out_copy;  /* SEQ copy output or nullptr                   */
    int32_t access;     /* AP_ACCESS_*                                  */
    uint64_t* ck;       /* per-thread checksums                         */
    unsigned long long* queue; /* AP_SEQ_QUEUE: next unit (zeroed per launch) */
};

__device__ __forceinline__ uint64_t uniform_off(const BenchArgs& a, uint32_t E, uint64_t t,
                                                uint64_t i) {
    return (ap::detail::sm64(a.seed ^ (t << 24) ^ i) % (a.span / E)) * E;
}

__device__ __forceinline__ uint64_t divergent_off(const BenchArgs& a, uint32_t E, uint64_t t,
                                                  uint64_t i) {
    const uint64_t npg = a.bytes / a.page;
    const uint64_t w = t >> 5, lane = t & 31;
    const uint64_t pg = (ap::detail::sm64(a.seed ^ (w << 24) ^ i) + lane * (npg / 32)) % npg;
    const uint64_t el =
        ap::detail::sm64(a.seed ^ (t << 24) ^ i ^ 0xD1B54A32D192ED03ull) % (a.page / E);
    return pg * a.page + el * E;
}

/* ------------------------------------------------------------ SEQ */
/* Loads are tiled TILE deep and double-buffered ("memory
 * tiling ... interleaves memory copy operations"): the next tile is issued
 * before the current one is consumed, so each warp keeps up to 2*TILE 512-B
 * requests in flight.  The apointer version and its raw twin run this same
 * loop; only the reader differs. */
#ifndef AP_TILE
#define AP_TILE 16
#endif
constexpr int TILE = AP_TILE;

template <class T>
__device__ __forceinline__ void consume(const BenchArgs& a, uint64_t off, const T& v,
                                        uint64_t& h) {
    if (a.out_copy) *reinterpret_cast<T*>(a.out_copy + off) = v;
    else h = fnv(h, v);
}
/* the same with the output kind fixed at compile time (per-access loops) */
template <bool COPY, class T>
__device__ __forceinline__ void consume_k(const BenchArgs& a, uint64_t off, const T& v,
                                          uint64_t& h) {
    if constexpr (COPY) *reinterpret_cast<T*>(a.out_copy + off) = v;
    else h = fnv(h, v);
}

/* raw-pointer reader with the apointer's interface (the twin) */
template <class T>
struct raw_reader {
    const T* p;
    template <int N>
    __device__ __forceinline__ void read_tile(T (&v)[N], int64_t stride) {
#pragma unroll
        for (int k = 0; k < N; ++k) v[k] = ap::detail::ld_data<T>(p + k * stride);
    }
    __device__ __forceinline__ raw_reader& operator+=(int64_t d) {
        p += d;
        return *this;
    }
    __device__ __forceinline__ T operator*() { return ap::detail::ld_data<T>(p); }
};

/* one unit, tiled: TILE loads issued before they are consumed */
template <class T, class R>
__device__ __forceinline__ void seq_unit(R& q, const BenchArgs& a, uint64_t e0, uint32_t per_unit,
                                         bool whole, uint64_t& h) {
    constexpr uint32_t E = sizeof(T);
    uint32_t j = 0;
    if (whole) {
        for (; j + TILE <= per_unit; j += TILE) {
            T v[TILE];
            q.read_tile(v, 32);
#pragma unroll
            for (int k = 0; k < TILE; ++k) consume(a, (e0 + 32ull * (j + k)) * E, v[k], h);
            q += 32 * TILE; /* after the values are used: no loads in flight at an unlink */
        }
        for (; j + TILE / 2 <= per_unit; j += TILE / 2) { /* short units (e.g. 4 KiB pages) */
            T v[TILE / 2];
            q.read_tile(v, 32);
#pragma unroll
            for (int k = 0; k < TILE / 2; ++k) consume(a, (e0 + 32ull * (j + k)) * E, v[k], h);
            q += 32 * (TILE / 2);
        }
    }
    for (; j < per_unit; ++j) {
        const uint64_t off = (e0 + 32ull * j) * E;
        if (off + E <= a.span) consume(a, off, (T)*q, h);
        q += 32;
    }
}

/* One unit, one access at a time: `v = *q; q += 32` (the paper's loop,
 * PAPER.md:310-316, 336), the same source for the apointer and its raw twin.
 *
 * Every access is its own dereference (its own translation check, its own
 * possible fault), so the only way for a warp to keep more than one load in
 * flight is to issue access j+D before it consumes access j: the loop keeps
 * the last D values in registers (AP_DEREF_PIPE; the pointer moves on before
 * the value it produced is used).  A check or a fault of access j+D then
 * never waits for the data of access j, and no loaded value is live across
 * the out-of-line fault path of the access that issues it (deref_slow reloads
 * lanes that were linked).  D = 1 is the plain loop. */
#ifndef AP_DEREF_PIPE
#define AP_DEREF_PIPE 8
#endif
template <class T, bool COPY, class R>
__device__ __forceinline__ void seq_unit_deref(R& q, const BenchArgs& a, uint64_t e0,
                                               uint32_t per_unit, bool whole, uint64_t& h) {
    constexpr uint32_t E = sizeof(T);
    constexpr int D = AP_DEREF_PIPE;
    uint32_t j = 0;
    if (D > 1 && whole && per_unit >= (uint32_t)D) {
        T v[D];
#pragma unroll
        for (int d = 0; d < D; ++d) {
            v[d] = *q;
            q += 32;
        }
        /* the ring holds accesses j .. j+D-1 */
        for (; j + 2 * D <= per_unit; j += D) {
#pragma unroll
            for (int d = 0; d < D; ++d) {
                const T nv = *q; /* access j + d + D */
                q += 32;
                consume_k<COPY>(a, (e0 + 32ull * (j + d)) * E, v[d], h);
                v[d] = nv;
            }
        }
#pragma unroll
        for (int d = 0; d < D; ++d) consume_k<COPY>(a, (e0 + 32ull * (j + d)) * E, v[d], h);
        j += D; /* per_unit % D accesses remain for the loop below */
    }
    for (; j < per_unit; ++j) {
        const uint64_t off = (e0 + 32ull * j) * E;
        if (off + E <= a.span) {
            const T v = *q;
            q += 32;
            consume_k<COPY>(a, off, v, h);
        } else {
            q += 32;
        }
    }
}

/* The per-access form keeps AP_DEREF_PIPE values per lane in registers
 * across the (ABI-called) fault path; built for AP_DEREF_MINB CTAs of 512
 * threads per SM (1 = 128 registers: 16 warps x 8 dereferences in flight
 * measured best; 2 = 64 registers, the paper's budget, fits a
 * ring of 4).  The raw twin runs the identical loop on a plain pointer at the
 * same launch. */
#ifndef AP_DEREF_MINB
#define AP_DEREF_MINB 1
#endif
template <class T, bool APTR, bool COPY>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_DEREF_MINB)
    k_seq_deref(const ap::dev_cache* __restrict__ c, uint32_t region, const BenchArgs a) {
    constexpr uint32_t E = sizeof(T);
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t w = t >> 5, lane = t & 31;
    const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nunits = (a.span + a.unit - 1) / a.unit;
    const uint32_t per_unit = a.unit / (32 * E);
    uint64_t h = FNV_BASIS;
    for (uint32_t pass = 0; pass < a.passes; ++pass) {
        for (uint64_t u = w; u < nunits; u += W) {
            const uint64_t e0 = u * (a.unit / E) + lane;
            const bool whole = (u + 1) * a.unit <= a.span;
            if constexpr (APTR) {
                ap::ptr<T> q = ap::gvmmap<T>(c, region, e0 * E);
                seq_unit_deref<T, COPY>(q, a, e0, per_unit, whole, h);
            } else {
                raw_reader<T> q{reinterpret_cast<const T*>(a.raw) + e0};
                seq_unit_deref<T, COPY>(q, a, e0, per_unit, whole, h);
            }
        }
    }
    if constexpr (!COPY) a.ck[t] = h;
}

/* AP_ACCESS_AHEAD: the tiled loop with a split-phase link.  The warp's next
 * unit is linked (ptr::link_begin) right after the current unit's last tile
 * is issued, so the PTE add travels with that tile's loads and the link
 * (link_finish) costs no extra round trip when the warp moves on.  Units
 * that are not whole or not a multiple of TILE deep take seq_unit. */
template <class T>
__device__ __forceinline__ void seq_ahead(const ap::dev_cache* c, uint32_t region,
                                          const BenchArgs& a, uint64_t w, uint64_t lane,
                                          uint64_t W, uint64_t nunits, uint32_t per_unit,
                                          uint64_t& h) {
    constexpr uint32_t E = sizeof(T);
    if (w >= nunits) return;
    const uint64_t per_warp = (nunits - w + W - 1) / W;
    const uint64_t total = per_warp * a.passes;
    const bool tiled = per_unit >= TILE && per_unit % TILE == 0;
    ap::ptr<T> q = ap::gvmmap<T>(c, region, (w * (a.unit / E) + lane) * E);
    uint64_t u = w;
    for (uint64_t k = 0; k < total; ++k) {
        const uint64_t e0 = u * (a.unit / E) + lane;
        uint64_t un = u + W;
        if (un >= nunits) un = w;
        const uint64_t next_off = (un * (a.unit / E) + lane) * E;
        if (!tiled || (u + 1) * a.unit > a.span) {
            seq_unit<T>(q, a, e0, per_unit, (u + 1) * a.unit <= a.span, h);
            q = ap::gvmmap<T>(c, region, next_off);
            u = un;
            continue;
        }
        uint32_t j = 0;
        for (; j + TILE < per_unit; j += TILE) {
            T v[TILE];
            q.read_tile(v, 32);
#pragma unroll
            for (int i = 0; i < TILE; ++i) consume(a, (e0 + 32ull * (j + i)) * E, v[i], h);
            q += 32 * TILE;
        }
        T v[TILE];
        q.read_tile(v, 32);
        ap::ptr<T> qn = ap::gvmmap<T>(c, region, next_off);
        const auto tk = qn.link_begin();
#pragma unroll
        for (int i = 0; i < TILE; ++i) consume(a, (e0 + 32ull * (j + i)) * E, v[i], h);
        q = static_cast<ap::ptr<T>&&>(qn); /* unlinks the finished unit */
        q.link_finish(tk);
        u = un;
    }
}

/* AP_ACCESS_PAIR: the tiled loop over two units at a time.  Both units'
 * pointers are linked together (two split-phase links: both PTE adds are in
 * flight at once, one round trip for two links), then the units are read
 * one after the other with the plain tile loop. */
template <class T>
__device__ __forceinline__ void seq_pair(const ap::dev_cache* c, uint32_t region,
                                         const BenchArgs& a, uint64_t w, uint64_t lane,
                                         uint64_t W, uint64_t nunits, uint32_t per_unit,
                                         uint64_t& h) {
    constexpr uint32_t E = sizeof(T);
    for (uint32_t pass = 0; pass < a.passes; ++pass) {
        for (uint64_t u = w; u < nunits; u += 2 * W) {
            const uint64_t u1 = u + W;
            const bool two = u1 < nunits && (u1 + 1) * a.unit <= a.span && (u + 1) * a.unit <= a.span;
            ap::ptr<T> q0 = ap::gvmmap<T>(c, region, (u * (a.unit / E) + lane) * E);
            if (!two) {
                seq_unit<T>(q0, a, u * (a.unit / E) + lane, per_unit, (u + 1) * a.unit <= a.span, h);
                if (u1 < nunits) {
                    ap::ptr<T> q1 = ap::gvmmap<T>(c, region, (u1 * (a.unit / E) + lane) * E);
                    seq_unit<T>(q1, a, u1 * (a.unit / E) + lane, per_unit,
                                (u1 + 1) * a.unit <= a.span, h);
                }
                continue;
            }
            ap::ptr<T> q1 = ap::gvmmap<T>(c, region, (u1 * (a.unit / E) + lane) * E);
            {
                const auto t0 = q0.link_begin();
                const auto t1 = q1.link_begin();
                q0.link_finish(t0);
                q1.link_finish(t1);
            }
            seq_unit<T>(q0, a, u * (a.unit / E) + lane, per_unit, true, h);
            q0.release();
            seq_unit<T>(q1, a, u1 * (a.unit / E) + lane, per_unit, true, h);
        }
    }
}

template <class T, bool APTR>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_SEQ_MINB)
    k_seq(const ap::dev_cache* __restrict__ c, uint32_t region, const BenchArgs a) {
    constexpr uint32_t E = sizeof(T);
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t w = t >> 5, lane = t & 31;
    const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nunits = (a.span + a.unit - 1) / a.unit;
    const uint32_t per_unit = a.unit / (32 * E);
    uint64_t h = FNV_BASIS;
    /* one pointer per thread walks its units: moving it to the next unit is
     * arithmetic, and the page it leaves is unlinked by the next unit's first
     * dereference (which can then reuse that frame, AP_POLICY_SEQUENTIAL) */
    [[maybe_unused]] ap::ptr<T> q;
    if constexpr (APTR) q = ap::gvmmap<T>(c, region, 0);
    for (uint32_t pass = 0; pass < a.passes; ++pass) {
        for (uint64_t u = w; u < nunits; u += W) {
            const uint64_t e0 = u * (a.unit / E) + lane;
            /* whole unit inside the span: tiled fast loop; else per element */
            const bool whole = (u + 1) * a.unit <= a.span;
            if constexpr (APTR) {
                q += (int64_t)(e0 * E - q.foff()) / (int64_t)E;
                if (a.access == AP_ACCESS_RANGE && whole) {
                    /* translate once for the unit, then stream plain loads
                     * through the linked translation (valid while q lives) */
                    const T* p = q.pin_range(32ull * E * (per_unit - 1) + E);
                    if (p) {
                        raw_reader<T> rr{p};
                        seq_unit<T>(rr, a, e0, per_unit, true, h);
                    } else {
                        seq_unit<T>(q, a, e0, per_unit, whole, h);
                    }
                } else {
                    seq_unit<T>(q, a, e0, per_unit, whole, h);
                }
            } else {
                raw_reader<T> q{reinterpret_cast<const T*>(a.raw) + e0};
                seq_unit<T>(q, a, e0, per_unit, whole, h);
            }
        }
    }
    if (!a.out_copy) a.ck[t] = h;
}

/* AP_SEQ_QUEUE: the k_seq stream with units handed out in order from a
 * device counter instead of round robin, so warps that hold frames keep
 * streaming while warps waiting for one hold a single unit (C1: 148 warps
 * over 64 frames; round robin leaves the last warps to finish alone).  The
 * next unit's index is fetched while the current one is read.  Copy output
 * only (the bytes land at their offsets whichever warp reads them). */
template <class T, bool APTR>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_SEQ_MINB)
    k_seq_queue(const ap::dev_cache* __restrict__ c, uint32_t region, const BenchArgs a) {
    constexpr uint32_t E = sizeof(T);
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t lane = t & 31;
    const uint64_t nunits = (a.span + a.unit - 1) / a.unit;
    const uint64_t total = nunits * a.passes;
    const uint32_t per_unit = a.unit / (32 * E);
    uint64_t h = FNV_BASIS;
    [[maybe_unused]] ap::ptr<T> q;
    if constexpr (APTR) q = ap::gvmmap<T>(c, region, 0);
    unsigned long long v = 0;
    if (lane == 0) v = atomicAdd(a.queue, 1ull);
    v = __shfl_sync(0xffffffffu, v, 0);
    while (v < total) {
        unsigned long long vn = 0;
        if (lane == 0) vn = atomicAdd(a.queue, 1ull);
        const uint64_t u = v % nunits;
        const uint64_t e0 = u * (a.unit / E) + lane;
        const bool whole = (u + 1) * a.unit <= a.span;
        if constexpr (APTR) {
            q += (int64_t)(e0 * E - q.foff()) / (int64_t)E;
            seq_unit<T>(q, a, e0, per_unit, whole, h);
        } else {
            raw_reader<T> q{reinterpret_cast<const T*>(a.raw) + e0};
            seq_unit<T>(q, a, e0, per_unit, whole, h);
        }
        v = __shfl_sync(0xffffffffu, vn, 0);
    }
}

/* The split-phase link experiments (AP_ACCESS_AHEAD, AP_ACCESS_PAIR) get a
 * kernel of their own, so adding them does not perturb ptxas's allocation of
 * k_seq's tile loop (tests/test_sass.py). */
template <class T>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_SEQ_MINB)
    k_seq_split(const ap::dev_cache* __restrict__ c, uint32_t region, const BenchArgs a) {
    constexpr uint32_t E = sizeof(T);
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t w = t >> 5, lane = t & 31;
    const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nunits = (a.span + a.unit - 1) / a.unit;
    const uint32_t per_unit = a.unit / (32 * E);
    uint64_t h = FNV_BASIS;
    if (a.access == AP_ACCESS_AHEAD) seq_ahead<T>(c, region, a, w, lane, W, nunits, per_unit, h);
    else seq_pair<T>(c, region, a, w, lane, W, nunits, per_unit, h);
    if (!a.out_copy) a.ck[t] = h;
}

/* AP_ACCESS_TMA (16-B elements, checksums): the SEQ stream staged through
 * shared memory with TMA bulk copies (cp.async.bulk + mbarrier) instead of a
 * register tile: TMA_ST stages of TMA_SB bytes per warp (12 KiB in flight
 * per warp, 192 KiB per CTA of 16 warps) and no loaded value in registers.
 * Apointer: each unit is pinned once (pin_range, a minor fault when
 * resident) when its first stage is issued and unlinked when its last stage
 * has been consumed, so the next unit's link overlaps the stages still in
 * flight (two units live at most: ptr[unit & 1]).  The raw twin runs the
 * same loop from a plain pointer.  Consumption order = the tiled kernel's,
 * so the checksums are identical. */
constexpr int TMA_ST = 6;
constexpr uint32_t TMA_SB = 2048;
constexpr int TMA_WARPS = AP_BENCH_THREADS / 32;

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

template <bool APTR>
__global__ void __launch_bounds__(AP_BENCH_THREADS, 1)
    k_seq_tma(const ap::dev_cache* __restrict__ c, uint32_t region, const BenchArgs a) {
    extern __shared__ __align__(128) uint8_t tma_smem[];
    __shared__ __align__(8) uint64_t mbar[TMA_WARPS][TMA_ST];
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const unsigned wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t w = t >> 5;
    const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nunits = a.span / a.unit;
    const uint32_t spu = a.unit / TMA_SB; /* stages per unit */
    uint8_t* buf = tma_smem + (size_t)wid * TMA_ST * TMA_SB;
    uint64_t h = FNV_BASIS;
    if (lane == 0) {
        for (int b = 0; b < TMA_ST; ++b)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[wid][b])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    const uint64_t per_warp = w < nunits ? (nunits - w + W - 1) / W : 0;
    const uint64_t total = per_warp * a.passes * spu; /* stages of this warp */
    [[maybe_unused]] ap::ptr<uint4> q[2];
    const uint8_t* ubase[2] = {nullptr, nullptr};
    auto issue = [&](uint64_t g) {
        const uint64_t k = g / spu, st = g % spu;
        const uint64_t u = w + (k % per_warp) * W;
        if (st == 0) {
            if constexpr (APTR) {
                q[k & 1] = ap::gvmmap<uint4>(c, region, u * a.unit);
                const uint4* p = q[k & 1].pin_range(a.unit);
                /* a failed pin (the fault path's watchdog; make_args rules out
                 * frame exhaustion) has set the sticky error: copy from the
                 * frame pool, always mapped, instead of address 0 */
                ubase[k & 1] = p ? reinterpret_cast<const uint8_t*>(p) : c->pool;
                /* frame data written by the generic proxy (fills), read by
                 * the async proxy (TMA) */
                asm volatile("fence.proxy.async.global;" ::: "memory");
            } else {
                ubase[k & 1] = a.raw + u * a.unit;
            }
        }
        if (lane == 0) {
            const uint32_t mb = smem_u32(&mbar[wid][g % TMA_ST]);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb),
                         "r"(TMA_SB) : "memory");
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                ::"r"(smem_u32(buf + (g % TMA_ST) * TMA_SB)), "l"(ubase[k & 1] + st * TMA_SB),
                "r"(TMA_SB), "r"(mb) : "memory");
        }
    };
    for (uint64_t g = 0; g < total && g < (uint64_t)TMA_ST; ++g) issue(g);
    for (uint64_t g = 0; g < total; ++g) {
        const int b = (int)(g % TMA_ST);
        const uint32_t parity = (uint32_t)((g / TMA_ST) & 1);
        const uint32_t mb = smem_u32(&mbar[wid][b]);
        uint32_t done = 0;
        while (!done)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                         : "=r"(done) : "r"(mb), "r"(parity) : "memory");
        const uint4* sv = reinterpret_cast<const uint4*>(buf + b * TMA_SB);
#pragma unroll
        for (int jj = 0; jj < (int)(TMA_SB / 512); ++jj) h = fnv(h, sv[jj * 32 + lane]);
        __syncwarp();
        if constexpr (APTR) {
            if (g % spu == spu - 1) q[(g / spu) & 1].release(); /* unit consumed */
        }
        if (g + TMA_ST < total) issue(g + TMA_ST);
    }
    a.ck[t] = h;
}

/* ------------------------------------------------------------ UNIFORM / DIVERGENT */
template <class T, int PAT, bool APTR>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_BENCH_MINB)
    k_random(const ap::dev_cache* __restrict__ c,
                                                  uint32_t region, const BenchArgs a) {
    constexpr uint32_t E = sizeof(T);
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint64_t h = FNV_BASIS;
    if constexpr (APTR) {
        ap::ptr<T> p = ap::gvmmap<T>(c, region, 0);
        uint64_t cur = 0;
        for (uint32_t i = 0; i < a.reads; ++i) {
            const uint64_t off = PAT == AP_UNIFORM ? uniform_off(a, E, t, i)
                                                   : divergent_off(a, E, t, i);
            p += ((int64_t)off - (int64_t)cur) / (int64_t)E; /* pointer arithmetic (S4) */
            cur = off;
            h = fnv(h, *p);
        }
    } else {
        const T* base = reinterpret_cast<const T*>(a.raw);
        for (uint32_t i = 0; i < a.reads; ++i) {
            const uint64_t off = PAT == AP_UNIFORM ? uniform_off(a, E, t, i)
                                                   : divergent_off(a, E, t, i);
            h = fnv(h, ap::detail::ld_data<T>(base + off / E));
        }
    }
    a.ck[t] = h;
}

template <class T, bool APTR>
cudaError_t launch_t(const ap_cache_s* c, ap_region_t region, const ap_bench_cfg* cfg,
                     const BenchArgs& a, cudaStream_t s) {
    switch (cfg->pattern) {
        case AP_SEQ:
            if (cfg->access == AP_ACCESS_DEREF) {
                if (a.out_copy)
                    k_seq_deref<T, APTR, true><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
                else
                    k_seq_deref<T, APTR, false><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
            }
            else if (APTR && (cfg->access == AP_ACCESS_AHEAD || cfg->access == AP_ACCESS_PAIR))
                k_seq_split<T><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
            else if (cfg->access == AP_ACCESS_TMA) {
                if constexpr (sizeof(T) == 16) {
                    const int smem = TMA_WARPS * TMA_ST * (int)TMA_SB;
                    cudaFuncSetAttribute(k_seq_tma<APTR>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                    k_seq_tma<APTR><<<cfg->grid, cfg->block, smem, s>>>(c->d_cache, region, a);
                }
            }
            else
                k_seq<T, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
            break;
        case AP_SEQ_QUEUE: {
            const cudaError_t e = cudaMemsetAsync(a.queue, 0, sizeof(unsigned long long), s);
            if (e != cudaSuccess) return e;
            k_seq_queue<T, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
            break;
        }
        case AP_UNIFORM:
            k_random<T, AP_UNIFORM, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
            break;
        default:
            k_random<T, AP_DIVERGENT, APTR><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region,
                                                                              a);
    }
    return cudaGetLastError();
}

template <bool APTR>
cudaError_t launch_m(const ap_cache_s* c, ap_region_t region, const ap_bench_cfg* cfg,
                     const BenchArgs& a, cudaStream_t s) {
    switch (cfg->elem_bytes) {
        case 4: return launch_t<uint32_t, APTR>(c, region, cfg, a, s);
        case 8: return launch_t<unsigned long long, APTR>(c, region, cfg, a, s);
        default: return launch_t<uint4, APTR>(c, region, cfg, a, s);
    }
}

int make_args(const ap_cache_s* c, ap_region_t region, const ap_bench_cfg* cfg, void* out,
              BenchArgs* a) {
    if (!ap_region_ok(c, region) || !cfg || !out) return AP_EINVAL;
    const uint32_t E = cfg->elem_bytes;
    if (E != 4 && E != 8 && E != 16) return AP_EINVAL;
    if (cfg->grid == 0 || cfg->block == 0 || cfg->block > AP_BENCH_THREADS || cfg->block % 32)
        return AP_EINVAL;
    if (cfg->mode != AP_MODE_APOINTER && cfg->mode != AP_MODE_RAW) return AP_EINVAL;
    if (cfg->mode == AP_MODE_RAW && !cfg->raw_base) return AP_EINVAL;
    const ap_region_host& rg = c->reg[region];
    *a = BenchArgs{};
    a->bytes = rg.bytes;
    a->seed = cfg->seed;
    a->raw = (const uint8_t*)cfg->raw_base;
    a->reads = cfg->reads_per_thread;
    a->passes = cfg->passes;
    a->unit = cfg->unit_bytes;
    a->page = cfg->page_bytes;
    a->span = cfg->span_bytes ? cfg->span_bytes : rg.bytes;
    a->access = cfg->access;
    if (cfg->access < AP_ACCESS_TILE || cfg->access > AP_ACCESS_TMA) return AP_EINVAL;
#ifdef AP_PT_HASH
    /* the split-phase link styles are not part of the hash-table ablation
     * (their relaxed early adds race with its probes) */
    if (cfg->mode == AP_MODE_APOINTER &&
        (cfg->access == AP_ACCESS_AHEAD || cfg->access == AP_ACCESS_PAIR))
        return AP_EINVAL;
#endif
    switch (cfg->pattern) {
        case AP_SEQ_QUEUE:
            /* copy output, tile access: the queue's unit order is dynamic */
            if (!cfg->out_copy || cfg->access != AP_ACCESS_TILE) return AP_EINVAL;
            a->queue = c->seq_queue;
            [[fallthrough]];
        case AP_SEQ:
            if (a->unit == 0 || a->unit % (32 * E) || a->span > rg.bytes) return AP_EINVAL;
            if (cfg->mode == AP_MODE_APOINTER && (c->page % a->unit)) return AP_EINVAL;
            if (cfg->out_copy) a->out_copy = (uint8_t*)out;
            else a->ck = (uint64_t*)out;
            /* TMA staging: 16-B checksums over whole units of whole stages,
             * at least as many stages per unit as are in flight */
            /* each warp pins up to two units at once (the next unit's pin
             * overlaps the current unit's stages): frames >= 2 per resident
             * warp, so no warp ever waits for a frame while pinning one */
            if (cfg->access == AP_ACCESS_TMA &&
                (E != 16 || cfg->out_copy || a->unit % TMA_SB || a->unit / TMA_SB < TMA_ST ||
                 a->span % a->unit || cfg->block > AP_BENCH_THREADS ||
                 (cfg->mode == AP_MODE_APOINTER && c->frames < rg.npages &&
                  c->frames < 2ull * std::min<uint64_t>(cfg->grid, c->num_sms) * (cfg->block / 32))))
                return AP_EINVAL;
            break;
        case AP_UNIFORM: /* offsets uniform over [0, span) (span 0 = the region) */
            if (a->span < E || a->span > rg.bytes) return AP_EINVAL;
            a->ck = (uint64_t*)out;
            break;
        case AP_DIVERGENT:
            if (a->page == 0 || (a->page & (a->page - 1)) || a->page < E ||
                rg.bytes / a->page < 32)
                return AP_EINVAL;
            a->ck = (uint64_t*)out;
            break;
        default: return AP_EINVAL;
    }
    return AP_OK;
}

}  // namespace

extern "C" int ap_bench_read(ap_cache_t c, ap_region_t region, const ap_bench_cfg* cfg,
                             void* out_dev, void* stream) {
    BenchArgs a;
    int rc = make_args(c, region, cfg, out_dev, &a);
    if (rc) return rc;
    ap_device_guard g(c->device);
    cudaError_t e = cfg->mode == AP_MODE_APOINTER
                        ? launch_m<true>(c, region, cfg, a, (cudaStream_t)stream)
                        : launch_m<false>(c, region, cfg, a, (cudaStream_t)stream);
    AP_CUDA_TRY(e);
    return AP_OK;
}

extern "C" int ap_bench_read_host(ap_cache_t c, ap_region_t region, const ap_bench_cfg* cfg,
                                  void* out_host, double* seconds) {
    if (!c || !cfg || !out_host) return AP_EINVAL;
    ap_device_guard g(c->device);
    const uint64_t nthreads = (uint64_t)cfg->grid * cfg->block;
    uint64_t out_bytes = nthreads * 8;
    if ((cfg->pattern == AP_SEQ || cfg->pattern == AP_SEQ_QUEUE) && cfg->out_copy)
        out_bytes = cfg->span_bytes ? cfg->span_bytes : c->reg[region].bytes;
    void* d = nullptr;
    AP_CUDA_TRY(cudaMalloc(&d, out_bytes));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0, 0);
    int rc = ap_bench_read(c, region, cfg, d, nullptr);
    if (rc == AP_OK) {
        cudaMemcpyAsync(out_host, d, out_bytes, cudaMemcpyDeviceToHost, 0);
        cudaEventRecord(e1, 0);
        if (cudaEventSynchronize(e1) != cudaSuccess) rc = AP_ECUDA;
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        if (seconds) *seconds = ms * 1e-3;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(d);
    return rc;
}

/* ------------------------------------------------------------------------
 * Latency microbenchmark (NEXT N4; the paper's Table I):
 * one warp, all lanes on one page, coalesced 4-B accesses; cycles per
 * operation from clock64() around each op, minus the cost of an empty
 * timing pair (the paper subtracts 16 cycles of measurement overhead). */
namespace {

__device__ __forceinline__ uint64_t clk() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%clock64;" : "=l"(t)::"memory");
    return t;
}
/* fold v into a live accumulator with a real instruction: the clock read
 * after it cannot issue before v has arrived */
#define SINK(v) asm volatile("add.u32 %0, %0, %1;" : "+r"(acc) : "r"((uint32_t)(v)) : "memory")
/* raw ops as volatile PTX so the compiler cannot hoist or fold them */
__device__ __forceinline__ uint32_t raw_ld(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void raw_add(const uint32_t*& p, int64_t d) {
    uint64_t a = (uint64_t)p;
    asm volatile("add.s64 %0, %0, %1;" : "+l"(a) : "l"(d * 4));
    p = (const uint32_t*)a;
}

__global__ void k_latency(const ap::dev_cache* __restrict__ c, uint32_t region, const uint32_t* raw,
                          int op, uint32_t reps, unsigned long long* out) {
    /* Each op is repeated `reps` times as a dependent chain between two
     * clock reads: the next read's address depends on the value just read
     * (an index inside the same page), so the reads cannot overlap and the
     * per-op time is the latency (pointer chasing).  Increments chain through
     * the pointer itself. */
    const unsigned lane = threadIdx.x & 31;
    ap::ptr<uint32_t> q = ap::gvmmap<uint32_t>(c, region, 4 * lane);
    const uint32_t* p = raw + lane;
    uint32_t acc = *q; /* links q (the page was prefilled: a minor fault) */
    acc += __ldcg(p);
    uint32_t v = acc;
    const uint64_t e0 = clk();
    SINK(v);
    const uint64_t e1 = clk();
    uint64_t t0 = 0, t1 = 0;
    switch (op) {
        case 0: /* raw read */
            t0 = clk();
            for (uint32_t i = 0; i < reps; ++i) v = raw_ld(p + 32 * (v & 7));
            SINK(v);
            t1 = clk();
            break;
        case 1: /* apointer read through the register translation */
            t0 = clk();
            for (uint32_t i = 0; i < reps; ++i) v = q[(int64_t)(32 * (v & 7))];
            SINK(v);
            t1 = clk();
            break;
        case 2: /* raw increment (stays in the page) */
            t0 = clk();
            for (uint32_t i = 0; i < reps; ++i) raw_add(p, (i & 1) ? -32 : 32);
            SINK((uint32_t)(uintptr_t)p);
            t1 = clk();
            break;
        case 3: /* apointer increment (stays in the page) */
            t0 = clk();
            for (uint32_t i = 0; i < reps; ++i) q += (i & 1) ? -32 : 32;
            SINK((uint32_t)q.x);
            t1 = clk();
            break;
        case 4: /* raw read + increment */
            t0 = clk();
            for (uint32_t i = 0; i < reps; ++i) {
                v = raw_ld(p + 32 * (v & 1));
                raw_add(p, (i & 1) ? -32 : 32);
            }
            SINK(v);
            t1 = clk();
            break;
        default: /* apointer read + increment */
            t0 = clk();
            for (uint32_t i = 0; i < reps; ++i) {
                v = q[(int64_t)(32 * (v & 1))];
                q += (i & 1) ? -32 : 32;
            }
            SINK(v);
            t1 = clk();
            break;
    }
    acc += v;
    if (lane == 0) {
        const uint64_t empty = e1 - e0;
        out[0] = (t1 - t0 - empty) / (reps ? reps : 1);
        out[1] = empty;
        out[2] = acc;
    }
}

}  // namespace

extern "C" int ap_bench_latency(ap_cache_t c, ap_region_t region, int op, uint32_t reps,
                                uint64_t* cycles) {
    if (!ap_region_ok(c, region) || op < 0 || op > 5 || !cycles) return AP_EINVAL;
    if (c->reg[region].bytes < c->page + 256) return AP_EINVAL;
    ap_device_guard g(c->device);
    int rc = ap_prefill(c, region, 0, 1, nullptr);
    if (rc) return rc;
    unsigned long long* d = nullptr;
    AP_CUDA_TRY(cudaMalloc(&d, 3 * sizeof(unsigned long long)));
    k_latency<<<1, 32>>>(c->d_cache, region, (const uint32_t*)c->pool, op, reps, d);
    cudaError_t e = cudaGetLastError();
    unsigned long long h[3] = {0, 0, 0};
    if (e == cudaSuccess) e = cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
    cudaFree(d);
    AP_CUDA_TRY(e);
    cycles[0] = h[0];
    cycles[1] = h[1];
    return AP_OK;
}

/* ------------------------------------------------------------------------
 * Writes through apointers (NEXT N3; Fig. 3 `*ptr = 25`) and
 * the apointer-to-apointer copy (the Table II copy kernel).
 * Value written at element e: low bytes of sm64(seed ^ e) (16-B elements:
 * sm64(seed ^ 2e), sm64(seed ^ (2e+1))).  Offsets: SEQ units as k_seq, or a
 * race-free permutation e = (t*R + i) * a mod M (perm_mult). */
namespace {

template <class T> __device__ __forceinline__ T wval(uint64_t seed, uint64_t e);
template <> __device__ __forceinline__ uint32_t wval<uint32_t>(uint64_t seed, uint64_t e) {
    return (uint32_t)ap::detail::sm64(seed ^ e);
}
template <> __device__ __forceinline__ unsigned long long wval<unsigned long long>(uint64_t seed,
                                                                                  uint64_t e) {
    return ap::detail::sm64(seed ^ e);
}
template <> __device__ __forceinline__ uint4 wval<uint4>(uint64_t seed, uint64_t e) {
    const uint64_t a = ap::detail::sm64(seed ^ (2 * e)), b = ap::detail::sm64(seed ^ (2 * e + 1));
    return make_uint4((uint32_t)a, (uint32_t)(a >> 32), (uint32_t)b, (uint32_t)(b >> 32));
}

/* permutation multiplier: the odd number nearest below 0.618*M that is
 * coprime with M (a bijection of [0, M) that scatters neighbours) */
__host__ __device__ inline uint64_t gcd_u64(uint64_t a, uint64_t b) {
    while (b) {
        const uint64_t t = a % b;
        a = b;
        b = t;
    }
    return a;
}
__host__ __device__ inline uint64_t perm_mult(uint64_t M) {
    uint64_t a = (uint64_t)(((unsigned __int128)M * 0x9E3779B97F4A7C15ull) >> 64) | 1;
    if (a >= M) a = 1;
    while (gcd_u64(a, M) != 1) a += 2;
    return a % M;
}
__device__ __forceinline__ uint64_t perm_idx(uint64_t k, uint64_t M, uint64_t A) {
    return ((k % M) * A) % M;
}

template <class T, int PAT>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_BENCH_MINB)
    k_write(const ap::dev_cache* __restrict__ c, uint32_t region, const BenchArgs a) {
    constexpr uint32_t E = sizeof(T);
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    if constexpr (PAT == AP_SEQ) {
        const uint64_t w = t >> 5, lane = t & 31;
        const uint64_t nunits = (a.span + a.unit - 1) / a.unit;
        const uint32_t per_unit = a.unit / (32 * E);
        for (uint64_t u = w; u < nunits; u += W) {
            const uint64_t e0 = u * (a.unit / E) + lane;
            ap::ptr<T> q = ap::gvmmap<T>(c, region, e0 * E);
            for (uint32_t j = 0; j < per_unit; ++j) {
                const uint64_t e = e0 + 32ull * j;
                if ((e + 1) * E <= a.span) q.store(wval<T>(a.seed, e));
                q += 32;
            }
        }
    } else {
        const uint64_t M = a.bytes / E;
        const uint64_t A = perm_mult(M);
        ap::ptr<T> p = ap::gvmmap<T>(c, region, 0);
        uint64_t cur = 0;
        for (uint32_t i = 0; i < a.reads; ++i) {
            const uint64_t e = perm_idx(t * a.reads + i, M, A);
            p += (int64_t)e - (int64_t)cur;
            cur = e;
            p.store(wval<T>(a.seed, e));
        }
    }
}

/* dst[e] = src[e] for e < span/E, both through apointers (the copy kernel
 * of PAPER.md:312: tiled reads, stores one element at a time). */
template <class T, bool APTR>
__global__ void __launch_bounds__(AP_BENCH_THREADS, AP_BENCH_MINB)
    k_copy(const ap::dev_cache* __restrict__ c, uint32_t src, uint32_t dst, const BenchArgs a) {
    constexpr uint32_t E = sizeof(T);
    constexpr int CT = TILE;
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t w = t >> 5, lane = t & 31;
    const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nunits = (a.span + a.unit - 1) / a.unit;
    const uint32_t per_unit = a.unit / (32 * E);
    if constexpr (!APTR) {
        /* raw twin: the same loop on plain pointers (src = raw, dst = raw + span) */
        const T* sp = reinterpret_cast<const T*>(a.raw);
        T* dp = reinterpret_cast<T*>(const_cast<uint8_t*>(a.raw) + a.span);
        for (uint64_t u = w; u < nunits; u += W) {
            const uint64_t e0 = u * (a.unit / E) + lane;
            uint32_t j = 0;
            if ((u + 1) * a.unit <= a.span) {
                for (; j + CT <= per_unit; j += CT) {
                    T v[CT];
#pragma unroll
                    for (int k = 0; k < CT; ++k) v[k] = ap::detail::ld_data<T>(sp + e0 + 32ull * (j + k));
#pragma unroll
                    for (int k = 0; k < CT; ++k) ap::detail::st_data<T>(dp + e0 + 32ull * (j + k), v[k]);
                }
            }
            for (; j < per_unit; ++j)
                if ((e0 + 32ull * j + 1) * E <= a.span)
                    ap::detail::st_data<T>(dp + e0 + 32ull * j, ap::detail::ld_data<T>(sp + e0 + 32ull * j));
        }
    } else {
        for (uint64_t u = w; u < nunits; u += W) {
            const uint64_t e0 = u * (a.unit / E) + lane;
            const bool whole = (u + 1) * a.unit <= a.span;
            ap::ptr<T> s = ap::gvmmap<T>(c, src, e0 * E);
            ap::ptr<T> d = ap::gvmmap<T>(c, dst, e0 * E);
            uint32_t j = 0;
            if (whole) {
                for (; j + CT <= per_unit; j += CT) {
                    T v[CT];
                    /* never hold one pin while the other pointer faults on a
                     * recycled cache (R-A19): drop it first under pressure */
                    if (!s.linked_all() && d.cache_pressure()) d.release();
                    s.read_tile(v, 32);
                    if (!d.store_ready() && s.cache_pressure()) s.release();
                    d.write_tile(v, 32);
                    s += 32 * CT;
                    d += 32 * CT;
                }
            }
            for (; j < per_unit; ++j) {
                if ((e0 + 32ull * j + 1) * E <= a.span) {
                    const T v = *s;
                    if (s.cache_pressure()) s.release();
                    d.store(v);
                    if (d.cache_pressure()) d.release();
                }
                s += 32;
                d += 32;
            }
        }
    }
}

template <class T>
cudaError_t launch_write(const ap_cache_s* c, ap_region_t region, const ap_bench_cfg* cfg,
                         const BenchArgs& a, cudaStream_t s) {
    if (cfg->pattern == AP_SEQ)
        k_write<T, AP_SEQ><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
    else
        k_write<T, AP_UNIFORM><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, region, a);
    return cudaGetLastError();
}

}  // namespace

extern "C" int ap_bench_write(ap_cache_t c, ap_region_t region, const ap_bench_cfg* cfg,
                              void* stream) {
    if (!ap_region_ok(c, region) || !cfg) return AP_EINVAL;
    if (!(c->reg[region].prot & AP_PROT_WRITE)) return AP_EINVAL;
    const uint32_t E = cfg->elem_bytes;
    if ((E != 4 && E != 8 && E != 16) || cfg->grid == 0 || cfg->block == 0 ||
        cfg->block > AP_BENCH_THREADS || cfg->block % 32)
        return AP_EINVAL;
    BenchArgs a{};
    a.bytes = c->reg[region].bytes;
    a.span = cfg->span_bytes ? cfg->span_bytes : a.bytes;
    a.unit = cfg->unit_bytes;
    a.reads = cfg->reads_per_thread;
    a.seed = cfg->seed;
    if (cfg->pattern == AP_SEQ) {
        if (a.unit == 0 || a.unit % (32 * E) || c->page % a.unit || a.span > a.bytes) return AP_EINVAL;
    } else if (cfg->pattern == AP_UNIFORM) {
        if ((uint64_t)cfg->grid * cfg->block * cfg->reads_per_thread > a.bytes / E) return AP_EINVAL;
        if (a.bytes / E > (1ull << 32)) return AP_ERANGE; /* perm_idx products stay in 64 bits */
    } else {
        return AP_EINVAL;
    }
    ap_device_guard g(c->device);
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    switch (E) {
        case 4: e = launch_write<uint32_t>(c, region, cfg, a, s); break;
        case 8: e = launch_write<unsigned long long>(c, region, cfg, a, s); break;
        default: e = launch_write<uint4>(c, region, cfg, a, s);
    }
    AP_CUDA_TRY(e);
    return AP_OK;
}

extern "C" int ap_bench_copy(ap_cache_t c, ap_region_t src, ap_region_t dst,
                             const ap_bench_cfg* cfg, void* stream) {
    if (!ap_region_ok(c, src) || !ap_region_ok(c, dst) || !cfg || src == dst) return AP_EINVAL;
    if (!(c->reg[dst].prot & AP_PROT_WRITE)) return AP_EINVAL;
    const uint32_t E = cfg->elem_bytes;
    if ((E != 4 && E != 8 && E != 16) || cfg->grid == 0 || cfg->block == 0 ||
        cfg->block > AP_BENCH_THREADS || cfg->block % 32)
        return AP_EINVAL;
    BenchArgs a{};
    a.bytes = c->reg[src].bytes;
    a.span = cfg->span_bytes ? cfg->span_bytes : a.bytes;
    a.unit = cfg->unit_bytes;
    if (a.unit == 0 || a.unit % (32 * E) || c->page % a.unit || a.span > a.bytes ||
        a.span > c->reg[dst].bytes)
        return AP_EINVAL;
    if (cfg->mode == AP_MODE_RAW) {
        if (!cfg->raw_base) return AP_EINVAL;
        a.raw = (const uint8_t*)cfg->raw_base; /* src; dst = raw_base + span */
    } else if (cfg->mode != AP_MODE_APOINTER) {
        return AP_EINVAL;
    }
    ap_device_guard g(c->device);
    cudaStream_t s = (cudaStream_t)stream;
    const bool aptr = cfg->mode == AP_MODE_APOINTER;
    switch (E) {
        case 4:
            if (aptr) k_copy<uint32_t, true><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, src, dst, a);
            else k_copy<uint32_t, false><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, src, dst, a);
            break;
        case 8:
            if (aptr) k_copy<unsigned long long, true><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, src, dst, a);
            else k_copy<unsigned long long, false><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, src, dst, a);
            break;
        default:
            if (aptr) k_copy<uint4, true><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, src, dst, a);
            else k_copy<uint4, false><<<cfg->grid, cfg->block, 0, s>>>(c->d_cache, src, dst, a);
    }
    AP_CUDA_TRY(cudaGetLastError());
    return AP_OK;
}
