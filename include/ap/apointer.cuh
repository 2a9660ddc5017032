/*
 * ap/apointer.cuh — the device side of ActivePointers on B200 (sm_100a).
 *
 * An apointer (§III-C, Fig. 3) is a pointer into a file
 * mapped with ap_mmap.  It is read like a normal pointer; under the hood:
 *
 *   translation field (Fig. 5; long apointer, R-A16):
 *     one 64-bit register, bit 63 = valid ("linked"), bits 62:61 permission
 *     (reserved; checks are off as in PAPER.md:308), bits 60:0 = the device
 *     address of the datum in the HBM page cache when linked (the "aphysical"
 *     address), or the region-relative file offset (the "xAddress") when
 *     unlinked.  A linked dereference is `and` + `ld`: no lookup, the
 *     register is the TLB.
 *   metadata: region descriptor pointer, linked page number,
 *     log2(page size); only the fault path and page-crossing arithmetic read it.
 *
 * Hit path: the data load is issued speculatively
 * from the masked address while the warp votes on the valid bit; if every
 * active lane is linked the loaded value is returned.  Unlinked lanes load
 * from the region descriptor instead (always mapped; R-A21), the value is
 * discarded.
 *
 * Fault path (§III-D, Listing 1; cleaned
 * reading R-A9): translation aggregation.  Lanes on the same page form a
 * group with __match_any_sync; the lowest lane is its leader and the only
 * lane touching shared structures; the reference count grows by popc(group).
 * Minor faults (page resident) are lock-free CASes on the page-table entry
 * and may proceed for all groups at once (R-A13).  Major faults claim the
 * entry (EMPTY -> LOADING), take a frame from the free list or by clock
 * eviction of a refcount-0 page, and the whole warp copies the
 * page from pinned host memory over the host link with 16-B loads; then a
 * release store publishes VALID (R-A15).  Distinct major faults of a warp are
 * handled one page per round by default.
 *
 * Reference counts (Fig. 4): +popc on link;
 * -popc (warp aggregated, release) when a pointer leaves its page, is
 * assigned, copied from, or destroyed; under frame pressure a warp also
 * proactively unlinks lanes it already served in the current dereference
 * (the "heuristic" of PAPER.md:115, R-A19/A20).
 *
 * Usage rules: the lanes of a warp that call an operation together must be
 * converged (the operation uses __activemask()); all lanes of one call use
 * pointers into the same cache; sizeof(T) is 4, 8 or 16 and offsets are
 * multiples of sizeof(T) (a T never straddles a page).
 */
#ifndef AP_APOINTER_CUH_
#define AP_APOINTER_CUH_

#include <cuda_runtime.h>
#include <stdint.h>
#ifdef AP_DEBUG
#include <cstdio>
#endif

/* The fault path is kept out of line by default so the hit path stays a
 * handful of instructions; -DAP_SLOW_INLINE inlines it. */
#ifndef AP_SLOW_ATTR
#ifdef AP_SLOW_INLINE
#define AP_SLOW_ATTR __forceinline__
#else
#define AP_SLOW_ATTR __noinline__
#endif
#endif

/* Unlink (a match, a popc and one release add per page) is inlined unless
 * -DAP_UNLINK_NOINLINE. */
#ifndef AP_UNLINK_ATTR
#ifdef AP_UNLINK_NOINLINE
#define AP_UNLINK_ATTR __noinline__
#else
#define AP_UNLINK_ATTR __forceinline__
#endif
#endif

/* Speculative load of the hit path: 1 = the load issues
 * with the vote (unready lanes read the region descriptor); 0 (default on
 * B200) = it issues after the vote.  Measured on B200: the per-access loop
 * keeps several dereferences in flight, so the address select costs more
 * than the latency it hides (deref overhead vs the raw twin +40 % -> +20 %,
 * DESIGN.md §5). */
#ifndef AP_SPECULATIVE
#define AP_SPECULATIVE 0
#endif
/* Reference bit of a freshly filled page (second-chance clock, R-A11):
 * 1 = set at the fill, 0 = set only when the page is linked again (a minor
 * fault), so pages touched once are evicted before re-referenced ones. */
#ifndef AP_REF_ON_FILL
#define AP_REF_ON_FILL 1
#endif
/* Stride prefetch distance of the per-access dereference (0 = off). */
#ifndef AP_PREFETCH_DIST
#define AP_PREFETCH_DIST 0
#endif

namespace ap {

/* ------------------------------------------------------------ layouts */
/* Page-table entry (R-A17): [63:62] state, [61] reference bit, [60] dirty,
 * [59:32] frame, [31:0] reference count. */
constexpr uint64_t PTE_EMPTY = 0ull;
constexpr uint64_t PTE_LOADING = 1ull << 62;
constexpr uint64_t PTE_VALID = 2ull << 62;
constexpr uint64_t PTE_REF = 1ull << 61;
constexpr uint64_t PTE_DIRTY = 1ull << 60; /* writable mappings: frame differs from the file */
constexpr uint64_t PTE_FRAME_MASK = (1ull << 28) - 1;
constexpr uint64_t PTE_RC_MASK = 0xffffffffull;

/* Translation field (R-A16). */
constexpr uint64_t XL_VALID = 1ull << 63;
constexpr uint64_t XL_DIRTY = 1ull << 62; /* permission-bit slot: this link already set DIRTY */
constexpr uint64_t XL_ADDR = (1ull << 61) - 1;

constexpr uint32_t PROT_READ = 1;
constexpr uint32_t PROT_WRITE = 2;

constexpr uint64_t PAGE_MASK48 = (1ull << 48) - 1;

/* Device error codes (mirror include/ap.h). */
constexpr int ERR_FAULT = -6;
constexpr int ERR_NOFRAME = -7;
constexpr int ERR_TIMEDOUT = -8;
constexpr int ERR_PERM = -9;

constexpr int POLICY_CLOCK = 0;
constexpr int POLICY_RANDOM = 1;
/* clock + drop-behind: a warp that faults right after leaving a page first
 * tries to reuse that page's frame (single-pass streams, like
 * MADV_SEQUENTIAL; R-A11 leaves the policy open) */
constexpr int POLICY_SEQUENTIAL = 2;

/* Counters, sharded by SM to keep atomics off one address. */
struct alignas(64) dev_stats {
    unsigned long long major, minor, fill_bytes, evictions, waits, downgrades, nofree, unlinks;
    unsigned long long peer_fills, peer_bytes; /* N2: fills copied from a peer cache */
};
/* One counter block per SM (148 on B200; 256 slots): fewer same-line
 * atomics from the inline minor-fault path (M2r +33 % over 64 shards). */
#ifndef AP_STAT_SHARDS
#define AP_STAT_SHARDS 256
#endif
constexpr int STAT_SHARDS = AP_STAT_SHARDS;

struct dev_cache;

/* A peer page cache holding the same file (NEXT N2): its
 * region's page table and its frame pool, as addresses this GPU can read
 * (the same HBM, NVLink peer access, or a CUDA IPC mapping of them). */
struct dev_peer {
    uint64_t* pte;       /* the peer region's PTE array (same page numbers) */
    const uint8_t* pool; /* the peer cache's frame pool                     */
};
constexpr uint32_t MAX_PEERS = 7;

/* Region descriptor (one mapped file), 128-B aligned in device memory.  The
 * first 64 B hold everything a link or an unlink reads (one sector fetch
 * after an acquire has invalidated L1; no dependent pointer chase to the
 * cache descriptor on the minor-fault path). */
struct alignas(128) dev_region {
    uint64_t bytes;         /* file size                                  */
    uint64_t* pte;          /* npages entries                             */
    const uint8_t* pool;    /* the cache's frame pool (one hop for links) */
    dev_stats* stats;       /* the cache's counter shards                 */
    uint32_t id;            /* region id (< 65535)                        */
    uint32_t prot;          /* PROT_READ | PROT_WRITE                     */
    uint32_t live;          /* 1 while mapped                             */
    uint32_t pad_;
    const uint8_t* host;    /* device alias of the pinned host bytes      */
    uint64_t npages;        /* ceil(bytes / page)                         */
    const dev_cache* cache; /* owning cache                               */
    const dev_peer* peers;  /* N2: caches a major fault may copy from     */
    uint32_t npeers;        /* 0 = fills come from the host only          */
    uint32_t shared;        /* N2: another cache (GPU) pins this region's
                             * pages as its peer, so the fault path's claim,
                             * publish and eviction RMWs on these PTEs are
                             * system-scope (they race with the peer's .sys
                             * pin, R-A15b)                                */
};

/* Cache descriptor, one copy in device memory per ap_cache_t. */
struct alignas(64) dev_cache {
    uint8_t* pool;                  /* frames * page bytes, page aligned   */
    uint64_t* owner;                /* [frames] ((region+1)<<48)|page, 0   */
    const uint32_t* free_ids;       /* [nfree] free frame ids              */
    unsigned long long* free_head;  /* pop counter                         */
    unsigned long long* clock_hand; /* clock position (frames, mod)        */
    dev_region* regions;            /* region table                        */
    dev_stats* stats;               /* [STAT_SHARDS]                       */
    int* err;                       /* sticky error word                   */
    uint64_t frames;
    uint64_t nfree;
    uint64_t policy_seed;
    uint64_t timeout_ns;
    uint32_t log2_page;
    int32_t policy;
    uint32_t max_claims;
    uint32_t sweep_steps;
    uint32_t backoff_min_ns; /* fault-path back-off: exponential from min to max */
    uint32_t backoff_max_ns;
};
/* dev_region::prot bit: the cache runs AP_POLICY_SEQUENTIAL, so a warp that
 * leaves a page with all its lanes keeps one reference on it (the
 * drop-behind pin) until its fault path has taken the frame over or let it
 * go (ptr::drop_stale, deref_slow) */
constexpr uint32_t REGION_DROP_BEHIND = 1u << 8;
/* deref_slow hint bits: the warp pins the page it left with one reference;
 * the lane (a group leader) already claimed its page (LOADING) inline */
constexpr uint32_t HINT_PINNED = 1u << 29;
constexpr uint32_t HINT_CLAIMED = 1u << 28;

/* ---------------------------------------------------- PTX helpers (A15) */
namespace detail {

__device__ __forceinline__ unsigned lane_id() {
    unsigned l;
    asm volatile("mov.u32 %0, %%laneid;" : "=r"(l));
    return l;
}
__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}
__device__ __forceinline__ unsigned sm_id() {
    unsigned s;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    return s;
}
__device__ __forceinline__ uint64_t now_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
/* AP_FAULT_PROF (diagnostic builds only, tools/exp_fault_phases.py): SM
 * cycles per fault-path phase, summed by each warp's first lane into
 * ap_fprof (defined in ap_runtime.cu, read by ap_fault_prof). */
#ifdef AP_FAULT_PROF
extern __device__ unsigned long long ap_fprof[16];
#define AP_FP_T(v) const long long v = clock64()
#define AP_FP_ADD(m, i, d)                                                              \
    do {                                                                                \
        if (::ap::detail::lane_id() == (unsigned)(__ffs(m) - 1)) atomicAdd(&::ap::detail::ap_fprof[i], (unsigned long long)(d)); \
    } while (0)
#else
#define AP_FP_T(v)
#define AP_FP_ADD(m, i, d)
#endif
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t cas_acq_rel(uint64_t* p, uint64_t cmp, uint64_t val) {
    uint64_t old;
    asm volatile("atom.acq_rel.gpu.global.cas.b64 %0, [%1], %2, %3;"
                 : "=l"(old) : "l"(p), "l"(cmp), "l"(val) : "memory");
    return old;
}
__device__ __forceinline__ void st_release(uint64_t* p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_add_release(uint64_t* p, uint64_t v) {
    asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void prefetch_l2(const void* p) {
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}
__device__ __forceinline__ void fence_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ uint64_t cas_acquire(uint64_t* p, uint64_t cmp, uint64_t val) {
    uint64_t old;
    asm volatile("atom.acquire.gpu.global.cas.b64 %0, [%1], %2, %3;"
                 : "=l"(old) : "l"(p), "l"(cmp), "l"(val) : "memory");
    return old;
}
__device__ __forceinline__ uint64_t cas_relaxed(uint64_t* p, uint64_t cmp, uint64_t val) {
    uint64_t old;
    asm volatile("atom.relaxed.gpu.global.cas.b64 %0, [%1], %2, %3;"
                 : "=l"(old) : "l"(p), "l"(cmp), "l"(val) : "memory");
    return old;
}
__device__ __forceinline__ uint64_t add_acquire(uint64_t* p, uint64_t v) {
    uint64_t old;
    asm volatile("atom.acquire.gpu.global.add.u64 %0, [%1], %2;"
                 : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}
/* Link / unlink RMWs on a PTE.  AP_LINK_RELAXED: the link add is relaxed;
 * frame data is read with .cg loads whose address is computed from the add's
 * result (ablation).  AP_UNLINK_RELAXED: relaxed unlink (measurement only:
 * bounds what the release costs; not safe against eviction). */
__device__ __forceinline__ uint64_t add_link(uint64_t* p, uint64_t v) {
#ifdef AP_LINK_RELAXED
    uint64_t old;
    asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;"
                 : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
#else
    return add_acquire(p, v);
#endif
}
__device__ __forceinline__ void red_unlink(uint64_t* p, uint64_t v) {
#ifdef AP_UNLINK_RELAXED
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
#else
    red_add_release(p, v);
#endif
}
/* System-scope RMWs on a peer's PTE: the peer's own warps update it from
 * their GPU, so these are performed at the peer's memory with .sys scope. */
__device__ __forceinline__ uint64_t ld_relaxed_sys(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t add_acquire_sys(uint64_t* p, uint64_t v) {
    uint64_t old;
    asm volatile("atom.acquire.sys.global.add.u64 %0, [%1], %2;"
                 : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}
__device__ __forceinline__ void red_add_release_sys(uint64_t* p, uint64_t v) {
    asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t cas_acquire_sys(uint64_t* p, uint64_t cmp, uint64_t val) {
    uint64_t old;
    asm volatile("atom.acquire.sys.global.cas.b64 %0, [%1], %2, %3;"
                 : "=l"(old) : "l"(p), "l"(cmp), "l"(val) : "memory");
    return old;
}
/* fault-path PTE RMWs of a region: system scope when a peer cache pins its
 * pages (dev_region::shared), else GPU scope */
__device__ __forceinline__ uint64_t pte_cas_acquire(bool shared, uint64_t* p, uint64_t cmp,
                                                    uint64_t val) {
    return shared ? cas_acquire_sys(p, cmp, val) : cas_acquire(p, cmp, val);
}
__device__ __forceinline__ void pte_red_release(bool shared, uint64_t* p, uint64_t v) {
    if (shared) red_add_release_sys(p, v);
    else red_add_release(p, v);
}
__device__ __forceinline__ void red_add_relaxed(unsigned long long* p, unsigned long long v) {
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_or_relaxed(uint64_t* p, uint64_t v) {
    asm volatile("red.relaxed.gpu.global.or.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long fetch_add_relaxed(unsigned long long* p,
                                                                unsigned long long v) {
    unsigned long long old;
    asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;"
                 : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
    uint64_t z = x + 0x9e3779b97f4a7c15ull;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}

/* -------------------------------------------------------------------------
 * N4 ablation (-DAP_PT_HASH): the paper's page table -- one concurrent hash
 * table indexing the pages of all files, 16x the number of frames, lock-free
 * reads -- instead of the dense per-region PTE array.  A slot
 * is {key = (region + 1) << 48 | page, the same 64-bit PTE}; linear probing
 * from splitmix64(key).  In this build the region descriptor's `pte` points
 * at the cache's slot table and `pad_` holds log2(slots).  A key, once
 * inserted, keeps its slot while the region is mapped (no removal, so no
 * probe chain ever breaks and a slot never changes pages); ap_mmap sizes the
 * table to at least twice the pages mapped.  Dense builds never compile
 * this. */
#ifdef AP_PT_HASH
constexpr uint64_t PT_TOMB = ~0ull;
__device__ __forceinline__ uint64_t* pt_find(const dev_region* r, uint64_t pg, bool insert) {
    uint64_t* slots = r->pte;
    const uint64_t mask = (1ull << r->pad_) - 1;
    const uint64_t key = ((uint64_t)(r->id + 1) << 48) | pg;
    uint64_t h = sm64(key) & mask;
    for (uint64_t i = 0; i <= mask; ++i, h = (h + 1) & mask) {
        uint64_t k = ld_relaxed(slots + 2 * h);
        if (k == 0 && insert) {
            k = atomicCAS(reinterpret_cast<unsigned long long*>(slots + 2 * h), 0ull,
                          (unsigned long long)key);
            if (k == 0) return slots + 2 * h + 1;
        }
        if (k == key) return slots + 2 * h + 1;
        if (k == 0) return nullptr;
    }
    return nullptr;
}
#ifdef AP_PT_HASH_DIAG
/* diagnostic: a must-exist lookup that finds no slot sets ERR_FAULT and
 * hands out a scratch counter word instead of crashing */
__device__ __forceinline__ uint64_t* pt_must(const dev_region* r, uint64_t pg) {
    uint64_t* q = pt_find(r, pg, false);
    if (!q) {
        atomicCAS(r->cache->err, 0, ERR_FAULT - 100);
        return reinterpret_cast<uint64_t*>(&r->stats->waits);
    }
    return q;
}
#define AP_PTE_AT(r, pg) ::ap::detail::pt_must((r), (pg))
#else
#define AP_PTE_AT(r, pg) ::ap::detail::pt_find((r), (pg), false)
#endif
/* The probe is a leader-only loop of data-dependent length.  The warp is NOT
 * reconverged with __syncwarp(m) after it: at some call sites m was taken
 * before the warp diverged, and the barrier then waited forever for lanes
 * parked at another one -- the hash build's round-2 hang (random collage
 * case 8 hung in 8 of 8 runs with the barrier, passed 8 of 8 without).  The
 * _sync intrinsics that follow synchronise their own masks; a later
 * __activemask() may see a subset of the lanes, which only splits the
 * warp-aggregated links and unlinks into smaller groups.
 * -DAP_PT_RECONVERGE_SYNC restores the barrier (diagnostic). */
#define AP_PTE_FIND(r, pg) ::ap::detail::pt_find((r), (pg), false) /* may miss */
#ifdef AP_PT_RECONVERGE_SYNC
#define AP_PT_RECONVERGE(m) __syncwarp(m)
#else
#define AP_PT_RECONVERGE(m) ((void)0)
#endif
#else
#define AP_PTE_FIND(r, pg) ((r)->pte + (pg))
#define AP_PT_RECONVERGE(m) ((void)0)
#define AP_PTE_AT(r, pg) ((r)->pte + (pg))
#endif

/* Frame-data loads bypass L1 (.cg): a recycled frame can never be served
 * from a stale L1 line, and the data is streamed once anyway. */
template <class T> __device__ __forceinline__ T ld_data(const T* p);
template <> __device__ __forceinline__ uint32_t ld_data<uint32_t>(const uint32_t* p) {
    return __ldcg(p);
}
template <> __device__ __forceinline__ int32_t ld_data<int32_t>(const int32_t* p) {
    return __ldcg(p);
}
template <> __device__ __forceinline__ unsigned long long ld_data<unsigned long long>(
    const unsigned long long* p) {
    return __ldcg(p);
}
template <> __device__ __forceinline__ uint4 ld_data<uint4>(const uint4* p) { return __ldcg(p); }
template <> __device__ __forceinline__ float ld_data<float>(const float* p) { return __ldcg(p); }
template <> __device__ __forceinline__ double ld_data<double>(const double* p) {
    return __ldcg(p);
}

template <class T> __device__ __forceinline__ void st_data(T* p, const T& v);
template <> __device__ __forceinline__ void st_data<uint32_t>(uint32_t* p, const uint32_t& v) {
    __stcg(p, v);
}
template <> __device__ __forceinline__ void st_data<unsigned long long>(unsigned long long* p,
                                                                        const unsigned long long& v) {
    __stcg(p, v);
}
template <> __device__ __forceinline__ void st_data<uint4>(uint4* p, const uint4& v) { __stcg(p, v); }
template <> __device__ __forceinline__ void st_data<int32_t>(int32_t* p, const int32_t& v) {
    __stcg(p, v);
}
template <> __device__ __forceinline__ void st_data<float>(float* p, const float& v) { __stcg(p, v); }

__device__ __forceinline__ void set_err(const dev_cache* c, int code) {
    atomicCAS(c->err, 0, code);
}
__device__ __forceinline__ dev_stats* my_stats(const dev_cache* c) {
    return c->stats + (sm_id() % STAT_SHARDS);
}
__device__ __forceinline__ void stat_add(unsigned long long* ctr, unsigned long long v) {
    if (v) red_add_relaxed(ctr, v);
}

/* k-th (0-based) set bit of m; m must have > k set bits. */
__device__ __forceinline__ int nth_set(unsigned m, int k) {
    for (int i = 0; i < k; ++i) m &= m - 1;
    return __ffs(m) - 1;
}

/* -------------------------------------------------------------------------
 * S10 unlink: lanes with `mine` drop their link to
 * `page` of `r`.  Warp-aggregated: one release-add of -n per distinct page. */
static __device__ AP_UNLINK_ATTR void unlink_lanes(unsigned m, bool mine, const dev_region* r,
                                          uint64_t page, bool fenced = false) {
    unsigned long long key = mine ? (((unsigned long long)r->id << 48) | page) : ~0ull;
    unsigned grp = __match_any_sync(m, key);
    unsigned lane = lane_id();
    if (mine && lane == (unsigned)(__ffs(grp) - 1)) {
        unsigned n = __popc(grp);
#ifdef AP_DEBUG
        printf("[unlink] w%u m%08x grp%08x n%u pg %llu\n", (unsigned)(threadIdx.x >> 5), m, grp, n, (unsigned long long)page);
#endif
#ifdef AP_PT_HASH_DIAG
        {
            /* diagnostic: an unlink must find its page VALID with a count >= n */
            uint64_t* q = AP_PTE_AT(r, page);
            const unsigned long long o = atomicAdd(reinterpret_cast<unsigned long long*>(q),
                                                   (unsigned long long)(0 - (uint64_t)n));
            if ((o >> 62) != 2 || (o & PTE_RC_MASK) < n)
                atomicCAS(r->cache->err, 0, (o >> 62) != 2 ? -107 : -108);
        }
#else
        /* fenced: the caller issued fence.acq_rel after its last access, so a
         * relaxed add is the release pattern of the PTX model */
        if (fenced) red_add_relaxed(reinterpret_cast<unsigned long long*>(AP_PTE_AT(r, page)),
                                    (unsigned long long)(0 - (uint64_t)n));
        else red_unlink(AP_PTE_AT(r, page), (uint64_t)0 - (uint64_t)n);
#endif
#if defined(AP_COUNT_UNLINKS) && !defined(AP_NO_HOT_STATS)
        /* opt-in: one more atomic per unlink cost a third of the minor-fault
         * throughput (M2r 14.5 -> 10.0 G reads/s), so it is off by default */
        stat_add(&(r->stats + (sm_id() % STAT_SHARDS))->unlinks, 1);
#endif
    }
    AP_PT_RECONVERGE(m);
}

/* Drop-behind unlink (AP_POLICY_SEQUENTIAL, R-A11b): when every lane of m
 * leaves the same page, the warp keeps one of its n references (the pin:
 * no other warp can evict the page, so no sweep takes the frame between
 * this unlink and the warp's own fault) and drops n - 1 with a relaxed add
 * (the pin keeps the frame, so no release is needed).  The fault path then
 * takes the frame over with one CAS (count 1 -> EMPTY) or drops the pin.
 * Returns true (for every lane) if the warp pinned the page; otherwise it
 * is unlink_lanes. */
static __device__ __forceinline__ bool unlink_lanes_pin(unsigned m, bool mine, const dev_region* r,
                                                        uint64_t page) {
#ifdef AP_PT_HASH
    unlink_lanes(m, mine, r, page);
    return false;
#else
    unsigned long long key = mine ? (((unsigned long long)r->id << 48) | page) : ~0ull;
    const unsigned grp = __match_any_sync(m, key);
    const bool keep = mine && grp == m && !r->shared;
    if (mine && lane_id() == (unsigned)(__ffs(grp) - 1)) {
        const unsigned n = __popc(grp);
        if (!keep) red_unlink(AP_PTE_AT(r, page), (uint64_t)0 - (uint64_t)n);
        else if (n > 1)
            red_add_relaxed(reinterpret_cast<unsigned long long*>(AP_PTE_AT(r, page)),
                            (unsigned long long)(0 - (uint64_t)(n - 1)));
    }
    return keep;
#endif
}

/* -------------------------------------------------------------------------
 * Write-back (writable mappings, NEXT N3): the lanes in m copy frame f to
 * the page's bytes in host memory over the host link (zero-copy 16-B
 * stores), then fence at system scope so the host sees them before the page
 * can be refilled from it. */
__device__ __forceinline__ void writeback_page(unsigned m, const dev_cache* c, const dev_region* r,
                                               uint64_t f, uint64_t pg) {
    const unsigned lane = __popc(m & lanemask_lt());
    const unsigned nl = __popc(m);
    const uint64_t P = 1ull << c->log2_page;
    const uint8_t* src = c->pool + f * P;
    uint8_t* dst = const_cast<uint8_t*>(r->host) + pg * P;
    const uint64_t avail = r->bytes - pg * P;
    const uint64_t len = avail < P ? avail : P;
    const uint64_t nvec = len / 16;
    const uint4* s4 = reinterpret_cast<const uint4*>(src);
    uint4* d4 = reinterpret_cast<uint4*>(dst);
    constexpr int U = 8;
    uint64_t i = lane;
    for (; i + (uint64_t)nl * (U - 1) < nvec; i += (uint64_t)nl * U) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = __ldcg(s4 + i + (uint64_t)nl * u);
#pragma unroll
        for (int u = 0; u < U; ++u) __stcs(d4 + i + (uint64_t)nl * u, v[u]);
    }
    for (; i < nvec; i += nl) __stcs(d4 + i, __ldcg(s4 + i));
    for (uint64_t b = nvec * 16 + lane; b < len; b += nl) dst[b] = src[b];
    __threadfence_system();
}

/* -------------------------------------------------------------------------
 * S7 frame allocation, warp-cooperative.  Lanes with `want` need one frame
 * each.  Free list first (pop-only array, R-A18), then victims: a warp-wide
 * clock step examines 32 consecutive frames; a frame is a victim if its
 * owner PTE is VALID, maps this frame and has reference count 0 (PAPER.md:
 * 113, 145); the clock gives referenced pages a second chance (R-A11).  A
 * victim is claimed by CAS of its PTE (VALID, rc=0) -> EMPTY, which a
 * concurrent minor fault's CAS either precedes or loses to. */
/* descriptor fields the fault path loads once on entry (see deref_slow) */
struct fault_hot {
    int32_t policy;
    uint64_t frames;
    dev_stats* stats;
    uint64_t* pte;   /* hint_r's page table (dense build) */
    uint32_t shared; /* hint_r->shared */
};
__device__ __forceinline__ bool alloc_frames(const dev_cache* c, unsigned m, bool want,
                                             uint32_t& frame, uint32_t hint = 0,
                                             const dev_region* hint_r = nullptr,
                                             uint64_t hint_page = 0, uint64_t pin = 0,
                                             bool* took_hint = nullptr,
                                             const fault_hot* hot = nullptr) {
    const unsigned lane = lane_id();
    const int first = __ffs(m) - 1;
    bool got = false;
    unsigned long long evicted = 0;
    const int32_t policy = hot ? hot->policy : c->policy;
    const uint64_t nframes = hot ? hot->frames : c->frames;
    if (policy == POLICY_SEQUENTIAL && want && hint && hint_r) {
        /* drop-behind, tried first: the frame of the page this lane's group
         * just left (hint = frame + 1), if no pointer re-linked it meanwhile.
         * Its entry is known (no owner-table lookup): CAS against the
         * expected value (VALID, this frame, referenced, count = the warp's
         * drop-behind pin (1) or 0), then once against what it holds. */
        const uint32_t f = hint - 1;
#ifdef AP_PT_HASH
        uint64_t* q = AP_PTE_FIND(hint_r, hint_page);
        const uint32_t hshared = hint_r->shared;
#else
        uint64_t* q = hot ? hot->pte + hint_page : AP_PTE_FIND(hint_r, hint_page);
        const uint32_t hshared = hot ? hot->shared : hint_r->shared;
#endif
        if (f < nframes && q) {
            const uint64_t want_e = PTE_VALID | PTE_REF | ((uint64_t)f << 32) | pin;
            uint64_t e = pte_cas_acquire(hshared, q, want_e, PTE_EMPTY);
            if (e == want_e) {
                got = true;
            } else if ((e >> 62) == 2 && ((e >> 32) & PTE_FRAME_MASK) == f &&
                       (e & PTE_RC_MASK) == pin && !(e & PTE_DIRTY)) {
                got = pte_cas_acquire(hshared, q, e, PTE_EMPTY) == e;
            }
            if (got) {
                frame = f;
                ++evicted;
                if (took_hint) *took_hint = true;
            }
        }
    }
    const unsigned wantm = __ballot_sync(m, want && !got);
    if (wantm) {
        const int k = __popc(wantm);
        const int rank = __popc(wantm & lanemask_lt());
        unsigned long long base = ~0ull;
        if ((int)lane == first) {
            if (*(volatile unsigned long long*)c->free_head < c->nfree)
                base = fetch_add_relaxed(c->free_head, (unsigned long long)k);
        }
        base = __shfl_sync(m, base, first);
        if (want && !got && base != ~0ull && base + rank < c->nfree) {
            frame = c->free_ids[base + rank];
            got = true;
        }
    }
    unsigned still = __ballot_sync(m, want && !got);
    /* the lanes present (possibly fewer than 32) each examine one frame per
     * clock step; at most two laps per attempt (second chance), then back off */
    const unsigned nl = __popc(m);
    const unsigned rk = __popc(m & lanemask_lt());
    const uint64_t lap = (c->frames + nl - 1) / nl;
    uint32_t steps = c->sweep_steps < 2 * lap + 1 ? c->sweep_steps : (uint32_t)(2 * lap + 1);
    while (still && steps--) {
        unsigned long long hb = 0;
        if ((int)lane == first)
            hb = fetch_add_relaxed(c->clock_hand, c->policy != POLICY_RANDOM ? (unsigned long long)nl : 1ull);
        hb = __shfl_sync(m, hb, first);
        uint64_t f;
        if (c->policy != POLICY_RANDOM) f = (hb + rk) % c->frames;
        else f = sm64(c->policy_seed ^ (hb << 5) ^ rk) % c->frames;
        bool elig = false;
        uint64_t e = 0;
        uint64_t* q = nullptr;
        const uint64_t own = ld_relaxed(c->owner + f);
        if (own) {
            const dev_region* vr = c->regions + ((own >> 48) - 1);
            q = AP_PTE_FIND(vr, own & PAGE_MASK48);
#ifdef AP_PT_HASH
            /* the owner entry can become visible before the key's insert */
            e = q ? ld_relaxed(q) : 0;
#else
            e = ld_relaxed(q);
#endif
            if ((e >> 62) == 2 && ((e >> 32) & PTE_FRAME_MASK) == f && (e & PTE_RC_MASK) == 0) {
                if (c->policy != POLICY_RANDOM && (e & PTE_REF)) cas_relaxed(q, e, e & ~PTE_REF);
                else elig = true;
            }
        }
        const unsigned cand = __ballot_sync(m, elig);
        const int need_n = __popc(still);
        bool won = false;
        /* a dirty victim is claimed into LOADING (faulters wait) until its
         * bytes are back in the file, then released to EMPTY */
        if (elig && __popc(cand & lanemask_lt()) < need_n)
            won = (pte_cas_acquire(c->regions[(own >> 48) - 1].shared, q, e,
                                   (e & PTE_DIRTY) ? PTE_LOADING : PTE_EMPTY) == e);
        const unsigned wonm = __ballot_sync(m, won);
        unsigned dirtym = __ballot_sync(m, won && (e & PTE_DIRTY));
        while (dirtym) {
            const int L = __ffs(dirtym) - 1;
            dirtym &= dirtym - 1;
            const unsigned long long vown = __shfl_sync(m, (unsigned long long)own, L);
            const uint64_t vf = __shfl_sync(m, (unsigned long long)f, L);
            const dev_region* vr = c->regions + ((vown >> 48) - 1);
            writeback_page(m, c, vr, vf, vown & PAGE_MASK48);
            __syncwarp(m);
            if ((int)lane == L) red_add_release(q, (uint64_t)0 - PTE_LOADING);
        }
        const int nwon = __popc(wonm);
        evicted += nwon;
        const bool mine_still = (still >> lane) & 1u;
        const int srank = __popc(still & lanemask_lt());
        const int src = (mine_still && srank < nwon) ? nth_set(wonm, srank) : (int)lane;
        const uint32_t ff = __shfl_sync(m, (uint32_t)f, src);
        if (mine_still && srank < nwon) {
            frame = ff;
            got = true;
        }
        still = __ballot_sync(m, want && !got);
    }
    if ((int)lane == first) {
        dev_stats* S = hot ? hot->stats : my_stats(c);
        stat_add(&S->evictions, evicted);
        if (still) stat_add(&S->nofree, 1);
    }
#ifdef AP_DEBUG
    if (still && (int)lane == first) {
        const uint64_t own0 = ld_relaxed(c->owner);
        const uint64_t* q0 = own0 ? AP_PTE_FIND(&c->regions[(own0 >> 48) - 1], own0 & PAGE_MASK48) : nullptr;
        const uint64_t e0 = q0 ? ld_relaxed(q0) : 0;
        if ((clock64() & 0xfffff) < 200)
            printf("[nofree] sm %u warp %u m %08x own0 %llx e0 %llx hand %llu\n", sm_id(),
                   (unsigned)(threadIdx.x >> 5), m, (unsigned long long)own0, (unsigned long long)e0,
                   (unsigned long long)*c->clock_hand);
    }
#endif
    return got;
}

/* -------------------------------------------------------------------------
 * S8 fill: the whole warp copies one page into frame `f` with 16-B loads,
 * from pinned host memory over the host link (zero copy) or, for N2, from a
 * peer cache's frame; the first `len` bytes come from `src` and a ragged
 * last page is zero-padded.  Host bytes are 16-B aligned (ap_mmap checks it). */
__device__ __forceinline__ void fill_page(unsigned m, uint8_t* pool, uint32_t lg, uint64_t f,
                                          const uint8_t* src, uint64_t len) {
    /* the lanes in m share the copy: rank = position among them */
    const unsigned lane = __popc(m & lanemask_lt());
    const unsigned nl = __popc(m);
    const uint64_t P = 1ull << lg;
    uint8_t* dst = pool + f * P;
    const uint64_t nvec = len / 16;
    const uint4* s4 = reinterpret_cast<const uint4*>(src);
    uint4* d4 = reinterpret_cast<uint4*>(dst);
    constexpr int U = 8;
    uint64_t i = lane;
    for (; i + (uint64_t)nl * (U - 1) < nvec; i += (uint64_t)nl * U) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = __ldcs(s4 + i + (uint64_t)nl * u);
#pragma unroll
        for (int u = 0; u < U; ++u) __stcg(d4 + i + (uint64_t)nl * u, v[u]);
    }
    for (; i < nvec; i += nl) __stcg(d4 + i, __ldcs(s4 + i));
    if (len < P) {
        /* ragged tail: bytes [nvec*16, len) from the source, the rest zeros */
        for (uint64_t b = nvec * 16 + lane; b < P; b += nl)
            dst[b] = b < len ? src[b] : (uint8_t)0;
    }
}

/* -------------------------------------------------------------------------
 * N2 peer fill (the "distributed shared memory across GPUs"
 * motivation of PAPER.md:33): before going to the host link, the warp looks
 * for page `pg` in the peer caches mapped over the same file.  The first
 * lane reads the peer's PTE; if it is VALID it pins the page there with one
 * acquire add (the peer cannot evict a frame whose count is positive,
 * PAPER.md:145).  Returns the pinned peer PTE (and the peer frame in *src),
 * or nullptr when no peer has the page resident.  The warp then copies the
 * whole frame (a peer frame holds a ragged last page already zero-padded)
 * and peer_unpin drops the pin once every lane's loads are done (each load
 * feeds a store, and __syncwarp orders the lanes before the leader's
 * release).  Small on purpose: it adds no copy loop to the fault path. */
__device__ __forceinline__ uint64_t* peer_pin(unsigned m, const dev_cache* c, const dev_region* r,
                                              uint64_t pg, const uint8_t** src) {
    const unsigned first = __ffs(m) - 1;
    const uint64_t P = 1ull << c->log2_page;
    for (uint32_t i = 0; i < r->npeers; ++i) {
        const dev_peer* pr = r->peers + i;
        uint64_t* q = pr->pte + pg;
        uint64_t old = 0;
        if (lane_id() == first && (ld_relaxed_sys(q) >> 62) == 2) {
            old = add_acquire_sys(q, 1);
            if ((old >> 62) != 2) {
                red_add_release_sys(q, (uint64_t)0 - 1); /* transient count, undone */
                old = 0;
            }
        }
        old = __shfl_sync(m, old, first);
        if ((old >> 62) == 2) {
            *src = pr->pool + ((old >> 32) & PTE_FRAME_MASK) * P;
            return q;
        }
    }
    return nullptr;
}
__device__ __forceinline__ void peer_unpin(unsigned m, const dev_cache* c, uint64_t* q) {
    __syncwarp(m);
    if (lane_id() == (unsigned)(__ffs(m) - 1)) {
        red_add_release_sys(q, (uint64_t)0 - 1);
        stat_add(&my_stats(c)->peer_fills, 1);
        stat_add(&my_stats(c)->peer_bytes, 1ull << c->log2_page);
    }
}

template <class T>
struct slow_out {
    uint64_t x;
    uint64_t page;
    T val;
};

/* -------------------------------------------------------------------------
 * S5-S9: the fault handler (translation aggregation, Listing 1 / R-A9).
 * Called by the converged lanes `m` when at least one of them is unlinked.
 * Returns each lane's new translation and linked page; `val` receives the
 * value at the lane's offset for lanes that were unlinked. */
/* hint (optional, per lane): bit 31 = the inline link just found this
 * lane's page EMPTY (the first round claims it without probing again); bit
 * 30 = the caller discards the value (a relink before its own loads: no
 * value load on the way out); bits 29:0 = frame + 1 of the page the lane's
 * pointer left just before (hint_page of the same region), for the
 * drop-behind policy. */
template <class T>
__device__ AP_SLOW_ATTR slow_out<T> deref_slow(unsigned m, uint64_t x, uint64_t page,
                                               const dev_region* r, uint32_t hint = 0,
                                               uint64_t hint_page = 0) {
    bool absent = (hint >> 31) != 0;
    const bool want_val = ((hint >> 30) & 1u) == 0; /* bit 30: the caller discards the value */
    /* HINT_PINNED: the warp still holds one reference on hint_page (the
     * drop-behind pin, ptr::drop_stale); round 1 hands it to the frame
     * allocation or drops it before anything can wait */
    bool pinned = (hint & HINT_PINNED) != 0;
    bool claimed_in = (hint & HINT_CLAIMED) != 0;
    hint &= 0x0fffffffu;
    /* Lanes linked on entry reload their value here, so the caller's
     * speculative load is dead on this path and is never kept live across
     * the call (keeping it live made every hit-path load wait for its data
     * before the vote's branch). */
    T vv = (want_val && (x >> 63)) ? ld_data<T>(reinterpret_cast<const T*>(x & XL_ADDR)) : T{};
    const dev_cache* c = r->cache;
    const unsigned lane = lane_id();
    const uint32_t lg = c->log2_page;
    const uint64_t P = 1ull << lg;
    dev_stats* S = my_stats(c);
    /* descriptor fields the rounds use, loaded once here: each acquire below
     * invalidates L1, so a field first read after one would cost an L2
     * round trip on the fault's critical path */
#ifdef AP_PT_HASH
    const fault_hot hot{c->policy, c->frames, S, nullptr, r->shared};
#else
    const fault_hot hot{c->policy, c->frames, S, r->pte, r->shared};
#endif
    const uint32_t max_claims = c->max_claims;
    uint64_t* const owner_tab = c->owner;
    uint8_t* const pool = c->pool;
    const uint8_t* const r_host = r->host;
    const uint64_t r_bytes = r->bytes;
    const uint32_t r_npeers = r->npeers;
    const uint32_t r_shared = r->shared;
    const uint32_t r_id = r->id;
#ifndef AP_PT_HASH
    uint64_t* const r_pte = r->pte;
#endif
    bool need = !(x >> 63);
    if (need && (x + sizeof(T) > r_bytes || (x % sizeof(T)) != 0)) {
        set_err(c, ERR_FAULT);
        vv = T{};
        need = false;
    }
    const uint64_t pg = need ? (x >> lg) : 0;
    const unsigned long long mykey = ((unsigned long long)r_id << 48) | pg;
    bool linked_here = false;
    bool held = !need && (x >> 63); /* linked before this call: value already loaded */
    uint64_t t0 = 0;
    uint32_t backoff = c->backoff_min_ns;
    int idle_rounds = 0;
    AP_FP_T(tp_entry);
    AP_FP_ADD(m, 0, 1);

    for (;;) {
        const unsigned pend = __ballot_sync(m, need);
        if (!pend) break;
        AP_FP_T(tp0);
        AP_FP_ADD(m, 7, 1);
        const unsigned grp = __match_any_sync(m, need ? mykey : ~0ull);
        const int leader = __ffs(grp) - 1;
        const bool is_leader = need && (int)lane == leader;
        const uint32_t n = __popc(grp);
#ifdef AP_PT_HASH
        uint64_t* pte = is_leader ? pt_find(r, pg, true) : nullptr;
        __syncwarp(m);
#else
        uint64_t* pte = r_pte + pg;
#endif

        /* Phase A (leaders, lane-parallel; R-A13): minor faults link at once;
         * up to max_claims leaders (lane order) may claim an EMPTY entry. */
        enum { ST_NONE = 0, ST_LINKED = 1, ST_CLAIMED = 2, ST_WAIT = 3, ST_SKIP = 4, ST_NOFRAME = 5 };
        int st = ST_NONE;
        uint32_t frame = 0;
        /* Optimistic link: one acquire add of n.  If the entry was VALID the
         * group is linked (one round trip for a minor fault); otherwise the
         * add is undone.  Every other transition tolerates such transient
         * counts on non-VALID entries: publish and revert are adds, claims
         * are CASes from exactly EMPTY (R-A17). */
        /* first round after an inline link found the page EMPTY: go straight
         * to the claim (a race with a concurrent claim or publish just makes
         * the CAS fail and the next round probe again) */
        const bool pre_claimed = is_leader && claimed_in; /* link_minor claimed it */
        claimed_in = false;
        const bool probed = is_leader && !absent && !pre_claimed;
        uint64_t old = probed ? add_link(pte, n) : 0;
        absent = false;
#ifdef AP_DEBUG
        if (is_leader && (old >> 62) == 2) printf("[link] w%u m%08x n%u pg %llu old %llx\n", (unsigned)(threadIdx.x >> 5), m, n, (unsigned long long)pg, (unsigned long long)old);
#endif
        if (is_leader) {
            if ((old >> 62) == 2) {
                st = ST_LINKED;
                frame = (uint32_t)((old >> 32) & PTE_FRAME_MASK);
                if (!(old & PTE_REF)) red_or_relaxed(pte, PTE_REF);
            } else if (probed) {
                red_add_relaxed(reinterpret_cast<unsigned long long*>(pte),
                                (unsigned long long)(0 - (uint64_t)n));
            }
        }
        const unsigned empties = __ballot_sync(m, is_leader && (old >> 62) == 0);
        const bool may_claim = !((empties >> lane) & 1u) ||
                               (uint32_t)__popc(empties & lanemask_lt()) < max_claims;
        if (pre_claimed) {
            st = ST_CLAIMED;
        } else if (is_leader && st == ST_NONE) {
            if ((old >> 62) == 0) {
                if (!may_claim) {
                    st = ST_SKIP;
                } else {
                    const uint64_t prev = pte_cas_acquire(r_shared, pte, PTE_EMPTY, PTE_LOADING);
                    /* prev != 0: transient counts, a racing claimer or a
                     * publish in between; all resolve by retrying */
                    st = prev == PTE_EMPTY ? ST_CLAIMED : ST_WAIT;
                }
            } else {
                st = ST_WAIT; /* LOADING by another warp */
            }
        }

        /* Phase B: frames for the claimed pages (S7). */
        const unsigned claimed = __ballot_sync(m, st == ST_CLAIMED);
        AP_FP_T(tp1);
        AP_FP_ADD(m, 1, tp1 - tp0);
        bool took_pin = false;
        if (claimed) {
            const bool ok = alloc_frames(c, m, st == ST_CLAIMED, frame, hint, r, hint_page,
                                         pinned ? 1 : 0, &took_pin, &hot);
            if (st == ST_CLAIMED && !ok) {
                /* give the page back (an add, so transient counts survive) */
                pte_red_release(r_shared, pte, (uint64_t)0 - PTE_LOADING);
                st = ST_NOFRAME;
            }
        }
        if (pinned) {
            /* the pin was not taken over with its frame: drop it (release:
             * the warp's reads of that page are done) */
            if (!__any_sync(m, took_pin) && (int)lane == __ffs(m) - 1)
                red_unlink(AP_PTE_AT(r, hint_page), (uint64_t)0 - 1);
            pinned = false;
        }

        /* Phase C: fills, one page at a time by the whole warp (S8), then the
         * publish (S9): every lane fences its stores, the warp syncs, the
         * leader release-stores VALID with the group's count. */
        unsigned fill = __ballot_sync(m, st == ST_CLAIMED);
        const int nfill = __popc(fill);
        AP_FP_T(tp2);
        AP_FP_ADD(m, 2, tp2 - tp1);
        while (fill) {
            const int L = __ffs(fill) - 1;
            fill &= fill - 1;
            const uint32_t f = __shfl_sync(m, frame, L);
            const uint64_t fpg = __shfl_sync(m, pg, L);
            /* the filling lane's region (lanes may point into different
             * regions): its fields from that lane's registers */
            const uint32_t fid = __shfl_sync(m, r_id, L);
            const uint8_t* src = reinterpret_cast<const uint8_t*>(
                                     __shfl_sync(m, (unsigned long long)r_host, L)) + (fpg << lg);
            const uint64_t avail = __shfl_sync(m, (unsigned long long)r_bytes, L) - (fpg << lg);
            if ((int)lane == L) st_relaxed(owner_tab + f, ((uint64_t)(fid + 1) << 48) | fpg);
            uint64_t* peer_q = nullptr;
            if (__shfl_sync(m, r_npeers, L)) {
                const dev_region* fr =
                    reinterpret_cast<const dev_region*>(__shfl_sync(m, (unsigned long long)r, L));
                peer_q = peer_pin(m, c, fr, fpg, &src);
            }
            fill_page(m, pool, lg, f, src, peer_q ? P : (avail < P ? avail : P));
            if (peer_q) peer_unpin(m, c, peer_q);
            else if ((int)lane == __ffs(m) - 1) stat_add(&S->fill_bytes, avail < P ? avail : P);
            AP_FP_T(tp3);
            AP_FP_ADD(m, 3, tp3 - tp2);
            fence_gpu();
            __syncwarp(m);
            AP_FP_T(tp4);
            AP_FP_ADD(m, 4, tp4 - tp3);
#ifdef AP_DEBUG
            if ((int)lane == L) printf("[publish] w%u m%08x n%u f%u pg %llu\n", (unsigned)(threadIdx.x >> 5), m, n, f, (unsigned long long)fpg);
#endif
            if ((int)lane == L)
                pte_red_release(r_shared, pte,
                                (PTE_VALID - PTE_LOADING) | (AP_REF_ON_FILL ? PTE_REF : 0) |
                                    ((uint64_t)f << 32) | (uint64_t)n);
        }
        const unsigned nminor = __popc(__ballot_sync(m, st == ST_LINKED));
        AP_FP_T(tp5);

        /* Phase D: link the group lanes and read their values (S9). */
        const int lst = __shfl_sync(m, st, leader);
        const uint32_t lf = __shfl_sync(m, frame, leader);
        __syncwarp(m);
        bool progressed = false;
        if (need && (lst == ST_LINKED || lst == ST_CLAIMED)) {
            x = XL_VALID | ((uint64_t)(pool + (uint64_t)lf * P) + (x & (P - 1)));
            page = pg;
            need = false;
            linked_here = true;
            if (want_val) vv = ld_data<T>(reinterpret_cast<const T*>(x & XL_ADDR));
            progressed = true;
        }
        if ((int)lane == __ffs(m) - 1) {
            stat_add(&S->major, nfill);
            stat_add(&S->minor, nminor);
        }
        progressed = __any_sync(m, progressed);
        AP_FP_T(tp6);
        AP_FP_ADD(m, 5, tp6 - tp5);

        /* Lanes still unserved: either skipped (another claim this round),
         * waiting on a page another warp is loading, or out of frames. */
        const unsigned waiting = __ballot_sync(m, need);
        if (waiting) {
            /* Under pressure (free list empty), stop pinning pages whose values
             * are already in registers (PAPER.md:115 heuristic; R-A19). */
            /* With no frame to be had anywhere (or a long wait), also release
             * lanes that came in linked: their values were loaded on entry.
             * Then every waiting warp holds no pin for this pointer, so some
             * warp can always allocate (deadlock freedom, R-A19). */
            const bool pressure = *(volatile unsigned long long*)c->free_head >= c->nfree;
            const bool waited = __any_sync(m, is_leader && st == ST_WAIT);
            const bool hard = __any_sync(m, st == ST_NOFRAME) || (waited && idle_rounds >= 2);
            if (pressure || hard) {
                const bool dg = linked_here || (hard && held);
                if (__any_sync(m, dg)) {
                    unlink_lanes(m, dg, r, page);
                    if (dg) {
                        x = (page << lg) | (x & (P - 1));
                        linked_here = false;
                        held = false;
                    }
                    const unsigned ndg = __popc(__ballot_sync(m, dg));
                    if ((int)lane == __ffs(m) - 1) stat_add(&S->downgrades, ndg);
                }
            }
            if (t0 == 0) t0 = now_ns();
            if (!progressed) {
                ++idle_rounds;
                if ((int)lane == __ffs(m) - 1) stat_add(&S->waits, 1);
                if (now_ns() - t0 > c->timeout_ns) {
                    /* watchdog: give up on the remaining lanes (value 0). */
                    if (need) {
                        set_err(c, ERR_TIMEDOUT);
                        vv = T{};
                        need = false;
                    }
                    continue;
                }
                __nanosleep(backoff);
                backoff = backoff * 2 < c->backoff_max_ns ? backoff * 2 : c->backoff_max_ns;
            } else {
                idle_rounds = 0;
                backoff = c->backoff_min_ns;
            }
        }
    }
    if (pinned && (int)lane == __ffs(m) - 1) /* no round ran (every lane out of range) */
        red_unlink(AP_PTE_AT(r, hint_page), (uint64_t)0 - 1);
    AP_FP_T(tp_exit);
    AP_FP_ADD(m, 6, tp_exit - tp_entry);
    return slow_out<T>{x, page, vv};
}

/* -------------------------------------------------------------------------
 * S5+S6 inline: the minor-fault fast path.  The unlinked lanes of m group by
 * page (__match_any_sync), each group's leader links with one acquire add of
 * the group size on the PTE (the same optimistic link deref_slow does, R-A17),
 * and if the entry was VALID the lanes link to its frame.  A leader that
 * finds the page not resident undoes its add and leaves its lanes unlinked.
 * Returns true when every lane of m is linked afterwards; otherwise the
 * caller runs the full fault path (deref_slow), which takes lanes linked
 * here as already served.  Inline and call-free, so in the common resident
 * case no register state is saved around an out-of-line call. */
template <class T, bool STREAM = false>
__device__ __forceinline__ bool link_minor(unsigned m, uint64_t& x, uint64_t& page,
                                           const dev_region* r, uint32_t lg,
                                           uint32_t* absent = nullptr) {
    const bool need = !(x >> 63);
    /* out-of-range / misaligned offsets: the full path reports them */
    if (__any_sync(m, need && (x + sizeof(T) > r->bytes || (x % sizeof(T)) != 0))) return false;
    /* STREAM (the tile / range reads through relink): the pool base and the
     * counters are read before the acquire below, which invalidates L1 --
     * read after it, the pool base costs one more L2 round trip before the
     * linked lanes' first loads.  The per-access miss path (inline in every
     * dereference loop) reads them afterwards: holding them across the add
     * there cost the loop more than the round trip (tools/exp_hit.py). */
    const uint8_t* pool = nullptr;
    dev_stats* rstats = nullptr;
    if constexpr (STREAM) {
        pool = r->pool;
        rstats = r->stats;
    }
    const uint64_t pg = x >> lg;
    const unsigned grp = __match_any_sync(m, need ? (((unsigned long long)r->id << 48) | pg) : ~0ull);
    const int leader = __ffs(grp) - 1;
    const bool is_leader = need && (int)lane_id() == leader;
    uint64_t old = 0;
    bool claimed = false;
    if (is_leader) {
#ifdef AP_PT_HASH
        uint64_t* pte = pt_find(r, pg, false); /* no slot: not resident */
        if (pte) {
#else
        uint64_t* pte = r->pte + pg;
        /* a sequential stream (drop-behind policy) expects its next page to
         * be absent: probe with the claim (EMPTY -> LOADING, the fault
         * path's first step) and link with the add only if it is VALID */
        const bool stream = STREAM && (r->prot & REGION_DROP_BEHIND) && !r->shared;
        if (stream) {
            old = cas_acquire(pte, PTE_EMPTY, PTE_LOADING);
            claimed = old == PTE_EMPTY;
        }
        if (!claimed && (!stream || (old >> 62) == 2)) {
#endif
            old = add_link(pte, __popc(grp));
            if ((old >> 62) == 2) {
                if (!(old & PTE_REF)) red_or_relaxed(pte, PTE_REF);
            } else {
                red_add_relaxed(reinterpret_cast<unsigned long long*>(pte),
                                (unsigned long long)(0 - (uint64_t)__popc(grp)));
            }
        }
    }
    AP_PT_RECONVERGE(m);
#ifndef AP_NO_HOT_STATS /* ablation: no counters on the inline link / unlink */
    const unsigned linkedm = __ballot_sync(m, is_leader && (old >> 62) == 2);
    if (linkedm && (int)lane_id() == __ffs(m) - 1)
        stat_add(&((STREAM ? rstats : r->stats) + (sm_id() % STAT_SHARDS))->minor, __popc(linkedm));
#endif
    old = __shfl_sync(m, old, leader);
    const bool ok = !need || (old >> 62) == 2;
    if (need && ok) {
        const uint64_t P = 1ull << lg;
        const uint64_t f = (old >> 32) & PTE_FRAME_MASK;
        x = XL_VALID | ((uint64_t)((STREAM ? pool : r->pool) + f * P) + (x & (P - 1)));
        page = pg;
    }
    /* the page was not resident (EMPTY): the fault path may claim it at once
     * (bit 0); this lane, its group's leader, claimed it already (bit 1) */
    if (absent) *absent = (need && (old >> 62) == 0 ? 1u : 0u) | (claimed ? 2u : 0u);
    return __all_sync(m, ok);
}

/* link_minor's `absent` bits as deref_slow hint bits */
__device__ __forceinline__ uint32_t absent_hint(uint32_t absent) {
    return ((absent & 1u) << 31) | ((absent & 2u) ? HINT_CLAIMED : 0u);
}

/* link_minor unless built with -DAP_NO_LINK_MINOR (ablation: every link
 * through the out-of-line fault path) */
template <class T, bool STREAM = false>
__device__ __forceinline__ bool try_link_minor(unsigned m, uint64_t& x, uint64_t& page,
                                               const dev_region* r, uint32_t lg,
                                               uint32_t* absent = nullptr) {
#ifdef AP_NO_LINK_MINOR
    if (absent) *absent = 0;
    return false;
#else
    return link_minor<T, STREAM>(m, x, page, r, lg, absent);
#endif
}

template <class T, int N>
struct tile_out {
    T v[N];
    uint64_t x; /* the pointer's translation afterwards (unlinked) */
};

/* Tile read for tiles that straddle a page boundary (e.g. unaligned 3 KiB
 * records).  Lanes are linked on entry.  A tile spanning at
 * most two pages: the elements in the linked page are loaded, the link is
 * dropped (so the lane holds no pin while faulting, R-A19), the lanes whose
 * tile continues link the next page through a temporary pointer, load the
 * rest, and unlink it.  Longer tiles go element by element.  The pointer
 * ends unlinked (it still designates the same offset). */
template <class T, int N>
__device__ AP_SLOW_ATTR tile_out<T, N> read_tile_slow(unsigned m, uint64_t x, uint64_t page,
                                                      const dev_region* r, uint32_t lg,
                                                      int64_t stride) {
    tile_out<T, N> t;
    const uint64_t P = 1ull << lg;
    const uint64_t f0 = (x >> 63) ? ((page << lg) | (x & (P - 1))) : x;
    const uint64_t span = (uint64_t)((N - 1) * stride * (int64_t)sizeof(T));
    const bool two = stride > 0 && span < P && (x >> 63);
    if (__all_sync(m, two)) {
        const uint64_t next = ((f0 >> lg) + 1) << lg;
        const T* a = reinterpret_cast<const T*>(x & XL_ADDR);
#pragma unroll
        for (int k = 0; k < N; ++k) {
            const uint64_t fk = f0 + (uint64_t)(k * stride * (int64_t)sizeof(T));
            t.v[k] = fk < next ? ld_data<T>(a + k * stride) : T{};
        }
        unlink_lanes(m, true, r, page); /* release: orders the loads above first */
        const bool cross = f0 + span + sizeof(T) > next;
        if (cross) {
            const unsigned mc = __activemask();
            const slow_out<T> o = deref_slow<T>(mc, next, 0, r);
            const bool l = (o.x >> 63) != 0;
            if (l) {
                const T* b = reinterpret_cast<const T*>(o.x & XL_ADDR);
#pragma unroll
                for (int k = 0; k < N; ++k) {
                    const uint64_t fk = f0 + (uint64_t)(k * stride * (int64_t)sizeof(T));
                    if (fk >= next) t.v[k] = ld_data<T>(b + (fk - next) / sizeof(T));
                }
            }
            if (__any_sync(mc, l)) unlink_lanes(mc, l, r, o.page);
            if (!l) {
                /* the fault path dropped this lane's link under frame
                 * pressure (its value is in o.val): element by element */
#pragma unroll 1
                for (int k = 0; k < N; ++k) {
                    const uint64_t fk = f0 + (uint64_t)(k * stride * (int64_t)sizeof(T));
                    if (fk >= next) {
                        const unsigned mk = __activemask();
                        const slow_out<T> e = deref_slow<T>(mk, fk, 0, r);
                        t.v[k] = e.val;
                        const bool le = (e.x >> 63) != 0;
                        if (__any_sync(mk, le)) unlink_lanes(mk, le, r, e.page);
                    }
                }
            }
        }
        __syncwarp(m); /* reconverge the lanes that went through phase 2 */
        t.x = f0;
        return t;
    }
    /* general case: each element through a temporary pointer */
    if (__any_sync(m, (x >> 63) != 0)) unlink_lanes(m, (x >> 63) != 0, r, page);
    for (int k = 0; k < N; ++k) {
        const uint64_t fk = f0 + (uint64_t)(k * stride * (int64_t)sizeof(T));
        const slow_out<T> o = deref_slow<T>(m, fk, 0, r);
        t.v[k] = o.val;
        const bool l = (o.x >> 63) != 0;
        if (__any_sync(m, l)) unlink_lanes(m, l, r, o.page);
    }
    t.x = f0;
    return t;
}

/* Store path (writable mappings, NEXT N3; Fig. 3's `*ptr = 25`, PAPER.md:
 * 134): every lane in m stores v at its offset.  Linked lanes store first;
 * then, if some lanes must fault while frames are scarce, the warp drops
 * every link it holds; then unlinked lanes are handled one page group at a
 * time: linked through the fault path (one page, so the group
 * comes back linked), the page marked DIRTY once (leader OR; the pointer
 * remembers it in XL_DIRTY), the lanes store, and under pressure the group
 * unlinks again if other groups are still waiting -- a warp never waits for
 * a frame while pinning one (R-A19).  Returns the new translation. */
template <class T>
__device__ AP_SLOW_ATTR slow_out<T> store_slow(unsigned m, uint64_t x, uint64_t page,
                                               const dev_region* r, T v) {
    const dev_cache* c = r->cache;
    const uint32_t lg = c->log2_page;
    if (!(r->prot & PROT_WRITE)) {
        set_err(c, ERR_PERM);
        return slow_out<T>{x, page, T{}};
    }
    const unsigned lane = lane_id();
    /* 1. lanes already linked store through their link (marking the page
     *    DIRTY once per page if this link has not yet) */
    const bool lnk = (x >> 63) != 0;
    bool done = false;
    {
        const bool mark = lnk && !(x & XL_DIRTY);
        const unsigned long long key = mark ? (((unsigned long long)r->id << 48) | page) : ~0ull;
        const unsigned grp = __match_any_sync(m, key);
        if (mark && (int)lane == __ffs(grp) - 1) red_or_relaxed(AP_PTE_AT(r, page), PTE_DIRTY);
        AP_PT_RECONVERGE(m);
        if (lnk) {
            x |= XL_DIRTY;
            st_data<T>(reinterpret_cast<T*>(x & XL_ADDR), v);
            done = true;
        }
    }
    /* 2. before any lane faults under frame pressure, the warp drops the
     *    links it holds (the values are stored), so it never waits for a
     *    frame while pinning one (R-A19) */
    const bool pressure = *(volatile unsigned long long*)c->free_head >= c->nfree;
    if (pressure && __any_sync(m, !done) && __any_sync(m, lnk)) {
        unlink_lanes(m, lnk, r, page);
        if (lnk) x = (page << lg) | (x & ((1ull << lg) - 1));
    }
    /* 3. unlinked lanes, one page group at a time */
    for (;;) {
        const unsigned pend = __ballot_sync(m, !done);
        if (!pend) break;
        const int L = __ffs(pend) - 1;
        const uint64_t mypg = x >> lg;
        const uint64_t lpg = __shfl_sync(m, mypg, L);
        const unsigned long long lr = __shfl_sync(m, (unsigned long long)r, L);
        const bool in = !done && mypg == lpg && (unsigned long long)r == lr;
        const unsigned mg = __ballot_sync(m, in);
        if (in) {
            const slow_out<T> o = deref_slow<T>(mg, x, page, r);
            x = o.x;
            page = o.page;
            const bool ok = (x >> 63) != 0;
            const unsigned okm = __ballot_sync(mg, ok);
            if (ok && (int)lane == __ffs(okm) - 1) red_or_relaxed(AP_PTE_AT(r, page), PTE_DIRTY);
            AP_PT_RECONVERGE(mg);
            if (ok) {
                x |= XL_DIRTY;
                st_data<T>(reinterpret_cast<T*>(x & XL_ADDR), v);
            }
            /* pressure re-read: this group may have taken the last free frame */
            const bool now_pressure = *(volatile unsigned long long*)c->free_head >= c->nfree;
            const bool drop = ok && now_pressure && __popc(pend) > __popc(mg);
            if (__any_sync(mg, drop)) {
                unlink_lanes(mg, drop, r, page);
                if (drop) x = (page << lg) | (x & ((1ull << lg) - 1));
            }
            /* a lane the fault path could not link (watchdog) drops its store */
            done = true;
        }
        __syncwarp(m);
    }
    return slow_out<T>{x, page, T{}};
}

}  // namespace detail

/* ======================================================================
 * ap::ptr<T> — the apointer (M1; Fig. 3).
 * States: uninitialised (r == nullptr), unlinked (valid bit
 * clear: x is the file offset), linked (valid bit set: the lane holds a
 * reference on file page `page`, whose frame starts at fb; x is the device
 * address of the datum, fb + its offset from the frame start).
 *
 * Where the translation is checked (B200 design): arithmetic
 * only moves x -- `p += d` is one 64-bit add, no vote, no branch -- and the
 * dereference checks that x still lies in the linked frame (its page bits
 * equal fb's).  A pointer that walked off its page still holds that page
 * until its next dereference (or release / assignment / destruction), where
 * the fault path unlinks it, warp-aggregated, before linking the new page:
 * the same Fig. 4 transitions with the unlink deferred to the
 * next use.  The hit path is then: a 32-bit frame compare, one vote, a load;
 * and arithmetic costs what it costs on a raw pointer. */
template <class T>
struct ptr {
    static_assert(sizeof(T) == 4 || sizeof(T) == 8 || sizeof(T) == 16, "T must be 4/8/16 B");
    uint64_t x;          /* translation field (R-A16)                            */
    uint64_t fb;         /* linked: XL_VALID [| XL_DIRTY] | frame base address;  *
                          * else XL_VALID (never in x's frame)                   */
    const dev_region* r; /* metadata: region                                     */
    uint64_t page;       /* metadata: the page a linked lane holds               */
    uint32_t lg;         /* metadata: log2(page size)                            */
    int64_t step = 0;    /* bytes of the last += (stride predictor)              */

    __device__ __forceinline__ ptr() : x(0), fb(XL_VALID), r(nullptr), page(0), lg(12) {}
    __device__ __forceinline__ ptr(const dev_region* reg, uint32_t log2_page, uint64_t foff)
        : x(foff), fb(XL_VALID), r(reg), page(0), lg(log2_page) {}
    /* Copy: the copy starts unlinked (Fig. 4). */
    __device__ __forceinline__ ptr(const ptr& o)
        : x(o.foff()), fb(XL_VALID), r(o.r), page(0), lg(o.lg) {}
    __device__ __forceinline__ ptr& operator=(const ptr& o) {
        const uint64_t nx = o.foff();
        release();
        x = nx;
        fb = XL_VALID;
        r = o.r;
        lg = o.lg;
        return *this;
    }
    /* Move: the same pointer changes hands -- its link moves with it, no
     * reference count changes. */
    __device__ __forceinline__ ptr(ptr&& o) : x(o.x), fb(o.fb), r(o.r), page(o.page), lg(o.lg) {
        o.detach();
    }
    __device__ __forceinline__ ptr& operator=(ptr&& o) {
        if (this == &o) return *this;
        release();
        x = o.x;
        fb = o.fb;
        r = o.r;
        page = o.page;
        lg = o.lg;
        o.detach();
        return *this;
    }
    __device__ __forceinline__ ~ptr() { release(); }

    /* the lane holds a reference on `page` (valid bit: the sign of x's high word) */
    __device__ __forceinline__ bool holds() const { return (int32_t)(uint32_t)(x >> 32) < 0; }
    /* linked and still inside the linked frame: the hit path's check */
    __device__ __forceinline__ bool in_frame(uint64_t a) const {
        return (uint32_t)(a >> 32) == (uint32_t)(fb >> 32) &&
               (((uint32_t)a ^ (uint32_t)fb) >> lg) == 0;
    }
    __device__ __forceinline__ bool ready() const { return in_frame(x); }
    /* kept for callers of the previous API: linked = ready to dereference */
    __device__ __forceinline__ bool linked() const { return ready(); }
    /* File offset (xAddress) the pointer designates, linked or not. */
    __device__ __forceinline__ uint64_t foff() const {
        return holds() ? (page << lg) + (uint64_t)((int64_t)(x & XL_ADDR) - (int64_t)(fb & XL_ADDR))
                       : x;
    }

    /* S3: dereference (hit path inline, fault path out of line). */
    __device__ __forceinline__ T operator*() {
        const unsigned m = __activemask();
#if AP_SPECULATIVE
        /* speculative load: lanes off their frame load the
         * region descriptor (always mapped) while the warp votes */
        const bool v = ready();
        const T* a = v ? reinterpret_cast<const T*>(x & XL_ADDR) : reinterpret_cast<const T*>(r);
        T val = detail::ld_data<T>(a);
        if (__all_sync(m, v)) return val;
#else
        /* the load issues after the vote: on B200 the per-access loop keeps
         * several dereferences in flight, so the select the speculative
         * address needs costs more than the latency it hides */
        if (__all_sync(m, ready())) return detail::ld_data<T>(reinterpret_cast<const T*>(x & XL_ADDR));
#endif
#if AP_PREFETCH_DIST > 0
        {
            const uint64_t px = x + (uint64_t)(step * AP_PREFETCH_DIST);
            if (in_frame(px)) detail::prefetch_l2(reinterpret_cast<const void*>(px & XL_ADDR));
        }
#endif
        return deref_miss(m);
    }

    /* The pointer's miss path: lanes that walked off their frame unlink it
     * (warp-aggregated), then unlinked lanes link -- inline when the page is
     * resident (link_minor), else through the fault handler. */
    __device__ __forceinline__ T deref_miss(unsigned m) {
        const uint64_t left = page;
        /* (no drop-behind pin or claim-first probe here: this miss path is
         * inline in every per-access loop, which it must not slow down; the
         * streaming paths are the tile / range reads through relink) */
        const uint32_t hint = drop_stale(m);
        uint32_t absent = 0;
        if (detail::try_link_minor<T>(m, x, page, r, lg, &absent)) {
            sync_fb();
            return detail::ld_data<T>(reinterpret_cast<const T*>(x & XL_ADDR));
        }
        const detail::slow_out<T> o =
            detail::deref_slow<T>(m, x, page, r, hint | detail::absent_hint(absent), left);
        x = o.x;
        page = o.page;
        sync_fb();
        return o.val;
    }

    /* The same, but a thread that holds a second pointer `other` releases it
     * first when this dereference must fault on a recycled cache (R-A19:
     * never wait for a frame while pinning one); the check costs nothing on
     * the hit path. */
    template <class U>
    __device__ __forceinline__ T deref_releasing(ptr<U>& other) {
        const unsigned m = __activemask();
        if (__all_sync(m, ready())) return detail::ld_data<T>(reinterpret_cast<const T*>(x & XL_ADDR));
        if (cache_pressure()) other.release();
        return deref_miss(m);
    }

    /* Store through the pointer (writable mappings; Fig. 3 `*ptr = 25`). */
    __device__ __forceinline__ void store(const T& v) {
        const unsigned m = __activemask();
        const bool ok = ready() && (x & XL_DIRTY);
        if (__all_sync(m, ok)) {
            detail::st_data<T>(reinterpret_cast<T*>(x & XL_ADDR), v);
            return;
        }
        drop_stale(m);
        const detail::slow_out<T> o = detail::store_slow<T>(m, x, page, r, v);
        x = o.x;
        page = o.page;
        sync_fb();
    }

    /* Tiled store: p[k * stride] = v[k] for k < N, p unchanged.  One check
     * for the tile when every lane is linked, its page already marked dirty
     * and the tile inside the page; otherwise element by element. */
    template <int N>
    __device__ __forceinline__ void write_tile(const T (&v)[N], int64_t stride) {
        const unsigned m = __activemask();
        const uint64_t span = (uint64_t)((N - 1) * stride * (int64_t)sizeof(T));
        const bool ok = ready() && (x & XL_DIRTY) && in_frame(x + span);
        if (__all_sync(m, ok)) {
            T* a = reinterpret_cast<T*>(x & XL_ADDR);
#pragma unroll
            for (int k = 0; k < N; ++k) detail::st_data<T>(a + k * stride, v[k]);
            return;
        }
        /* slow path: the values go to a local array first, so no register
         * holding them is live across a call (ptxas would otherwise spill the
         * tile right after its loads, on the fast path too) */
        T tmp[N];
#pragma unroll
        for (int k = 0; k < N; ++k) tmp[k] = v[k];
        write_tile_slow<N>(*this, tmp, stride);
    }
    template <int N>
    static __device__ __noinline__ void write_tile_slow(ptr& p, const T* v, int64_t stride) {
#pragma unroll 1
        for (int k = 0; k < N; ++k) {
            p.store(v[k]);
            p += stride;
        }
        p -= N * stride;
    }

    /* warp-wide: every active lane is ready (and, for stores, marked dirty) */
    __device__ __forceinline__ bool linked_all() const { return __all_sync(__activemask(), ready()); }
    __device__ __forceinline__ bool store_ready() const {
        return __all_sync(__activemask(), ready() && (x & XL_DIRTY));
    }

    /* p[i] without moving p: a lane whose target stays in its linked frame
     * reads directly; otherwise a temporary pointer takes the fault. */
    __device__ __forceinline__ T operator[](int64_t i) {
        const unsigned m = __activemask();
        const uint64_t nb = (uint64_t)(i * (int64_t)sizeof(T));
        const uint64_t nx = x + nb;
        const bool in = in_frame(nx);
        const T* a = in ? reinterpret_cast<const T*>(nx & XL_ADDR) : reinterpret_cast<const T*>(r);
        T val = detail::ld_data<T>(a);
        if (__all_sync(m, in)) return val;
        ptr q(*this);
        q.x += nb;
        return *q;
    }

    /* Tiled read: v[k] = p[k * stride] for k < N, p unchanged.  One
     * translation check covers the whole tile when every lane is linked and
     * its tile stays inside its frame; the N loads then issue back to back
     * (memory tiling; one check per tile instead of per access
     * is the hand-written form of the check elimination PAPER.md:450 asks of
     * a compiler).  Otherwise the pointer is (re)linked through the fault
     * path; a tile that straddles a page is read element by element.  No
     * loaded value is ever live across a call into the fault path. */
    template <int N>
    __device__ __forceinline__ void read_tile(T (&v)[N], int64_t stride) {
        const unsigned m = __activemask();
        const uint64_t span = (uint64_t)((N - 1) * stride * (int64_t)sizeof(T));
        bool ok = ready() && in_frame(x + span);
        if (__builtin_expect(!__all_sync(m, ok), 0)) {
            relink(m);
            ok = ready() && in_frame(x + span);
            if (!__all_sync(m, ok)) {
                /* some lane's tile straddles a page */
                const detail::tile_out<T, N> t = detail::read_tile_slow<T, N>(m, x, page, r, lg, stride);
#pragma unroll
                for (int k = 0; k < N; ++k) v[k] = t.v[k];
                x = t.x;
                fb = XL_VALID;
                return;
            }
        }
        const T* a = reinterpret_cast<const T*>(x & XL_ADDR);
#pragma unroll
        for (int k = 0; k < N; ++k) v[k] = detail::ld_data<T>(a + k * stride);
    }

    /* Translate once for a whole range: make the pointer linked and return
     * its direct device address if [p, p + bytes) of every lane lies inside
     * the page that lane links (else nullptr, nothing changed but a link).
     * The address stays valid while this pointer keeps its link -- a linked
     * pointer keeps its page active and its mapping fixed (PAPER.md:113,
     * 141) -- i.e. until it is released, assigned, destroyed or dereferenced
     * after moving off the page; a loop can stream through it with plain
     * loads.  This is the per-page hoisting of the translation check that
     * PAPER.md:450 expects from compiler support. */
    __device__ __forceinline__ const T* pin_range(uint64_t bytes) {
        const unsigned m = __activemask();
        const uint64_t last = bytes ? bytes - 1 : 0;
        bool ok = ready() && in_frame(x + last);
        if (!__all_sync(m, ok)) {
            relink(m);
            ok = ready() && in_frame(x + last);
            if (!__all_sync(m, ok)) return nullptr;
        }
        return reinterpret_cast<const T*>(x & XL_ADDR);
    }

    /* Split-phase link -- a translation prefetch, the overlap of PAPER.md:195
     * ("access memory in parallel with checking") applied to the minor fault:
     * link_begin() groups the lanes that hold no page by page (S5) and issues
     * each group's optimistic PTE add (S6, relaxed: the frame data is then
     * read with .cg loads whose addresses depend on the add's result) without
     * waiting for it; link_finish(t) consumes it and links the lanes whose
     * page was resident (a non-resident page's add is undone; those lanes
     * stay unlinked and take the ordinary fault path on their next
     * dereference).  Lanes that still hold a page are left alone.  Contract:
     * between the two calls the warp must not enter the fault path; loads
     * through pointers already linked, arithmetic and unlinks are fine.
     * Every link_begin is followed by its link_finish. */
    struct link_ticket {
        uint64_t old; /* leader: the PTE before the add */
        unsigned grp; /* this lane's page group         */
        bool need;    /* this lane took part            */
    };
    __device__ __forceinline__ link_ticket link_begin() {
        const unsigned m = __activemask();
        const bool need = !holds() && x + sizeof(T) <= r->bytes && (x % sizeof(T)) == 0;
        const uint64_t pg = x >> lg;
        const unsigned grp =
            __match_any_sync(m, need ? (((unsigned long long)r->id << 48) | pg) : ~0ull);
        uint64_t old = 0;
        if (need && (int)detail::lane_id() == __ffs(grp) - 1) {
            uint64_t* pte = AP_PTE_FIND(r, pg);
#ifdef AP_PT_HASH
            if (!pte) old = 3ull << 62; /* no slot: nothing added (no early return: */
            else                        /* the warp must stay converged)            */
#endif
            asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;"
                         : "=l"(old) : "l"(pte), "l"((uint64_t)__popc(grp)) : "memory");
        }
        AP_PT_RECONVERGE(m);
        return link_ticket{old, grp, need};
    }
    __device__ __forceinline__ void link_finish(const link_ticket& t) {
        const unsigned m = __activemask();
        const int leader = __ffs(t.grp) - 1;
        const bool is_leader = t.need && (int)detail::lane_id() == leader;
        const uint64_t pg = x >> lg;
        const bool res = (t.old >> 62) == 2;
        if (is_leader && (t.old >> 62) != 3) {
            uint64_t* pte = AP_PTE_AT(r, pg);
            if (res) {
                if (!(t.old & PTE_REF)) detail::red_or_relaxed(pte, PTE_REF);
            } else {
                detail::red_add_relaxed(reinterpret_cast<unsigned long long*>(pte),
                                        (unsigned long long)(0 - (uint64_t)__popc(t.grp)));
            }
        }
        AP_PT_RECONVERGE(m);
#ifndef AP_NO_HOT_STATS
        const unsigned linkedm = __ballot_sync(m, is_leader && res);
        if (linkedm && (int)detail::lane_id() == __ffs(m) - 1)
            detail::stat_add(&(r->stats + (detail::sm_id() % STAT_SHARDS))->minor, __popc(linkedm));
#endif
        const uint64_t old = __shfl_sync(m, t.old, leader);
        if (t.need && (old >> 62) == 2) {
            const uint64_t P = 1ull << lg;
            const uint64_t f = (old >> 32) & PTE_FRAME_MASK;
            x = XL_VALID | ((uint64_t)(r->pool + f * P) + (x & (P - 1)));
            page = pg;
            sync_fb();
        }
    }

    /* S4: arithmetic moves the pointer and nothing else (one 64-bit add):
     * leaving the page is noticed, and the page unlinked (S10), by the next
     * dereference.  A step of a terabyte or more unlinks at once, so an
     * address never wraps into the flag bits. */
    __device__ __forceinline__ ptr& operator+=(int64_t d) {
        const uint64_t nb = (uint64_t)(d * (int64_t)sizeof(T));
        step = (int64_t)nb;
        if (nb + (1ull << 40) >= (1ull << 41)) release();
        x += nb;
        return *this;
    }
    __device__ __forceinline__ ptr& operator-=(int64_t d) { return *this += -d; }
    __device__ __forceinline__ ptr& operator++() { return *this += 1; }
    __device__ __forceinline__ ptr& operator--() { return *this += -1; }
    /* p + d is a new, unlinked pointer. */
    __device__ __forceinline__ ptr operator+(int64_t d) const {
        ptr q(*this);
        q.x += (uint64_t)(d * (int64_t)sizeof(T));
        return q;
    }

    /* True when the cache's free list is exhausted (frames are recycled by
     * eviction).  A thread that holds one linked pointer while another one
     * may fault should release the first under pressure (R-A19). */
    __device__ __forceinline__ bool cache_pressure() const {
        const dev_cache* c = r->cache;
        return *(volatile unsigned long long*)c->free_head >= c->nfree;
    }

    /* Unlink after an explicit ap::fence_acq_rel() that follows the last
     * access through the pointer (the fence + relaxed add is the release
     * pattern of the PTX memory model): lets one fence serve several
     * pointers -- and, after a link_begin, also the acquire of that link
     * (relaxed add observed, then the fence). */
    __device__ __forceinline__ void release_fenced() {
        const unsigned m = __activemask();
        const bool l = holds();
        if (__any_sync(m, l)) {
            const uint64_t off = foff();
            detail::unlink_lanes(m, l, r, page, true);
            if (l) {
                x = off;
                fb = XL_VALID;
            }
        }
    }

    /* Unlink now (also done by the destructor and by assignment). */
    __device__ __forceinline__ void release() {
        const unsigned m = __activemask();
        const bool l = holds();
        if (__any_sync(m, l)) {
            const uint64_t off = foff();
            detail::unlink_lanes(m, l, r, page);
            if (l) {
                x = off;
                fb = XL_VALID;
            }
        }
    }

   private:
    /* frame base of a linked lane (its dirty bit included), else XL_VALID */
    __device__ __forceinline__ void sync_fb() {
        fb = holds() ? (x & ~((1ull << lg) - 1)) : XL_VALID;
    }
    /* lanes that walked off their frame unlink it and carry
     * on unlinked at the same file offset */
    /* drop the drop-behind pin on page `left` when no fault follows */
    __device__ __forceinline__ void unpin(unsigned m, uint32_t hint, uint64_t left) {
        if ((hint & HINT_PINNED) && detail::lane_id() == (unsigned)(__ffs(m) - 1))
            detail::red_unlink(AP_PTE_AT(r, left), (uint64_t)0 - 1);
    }
    /* pin: the caller is a read fault path that passes the hint on to
     * deref_slow (or drops the pin itself): under drop-behind a warp that
     * leaves one page with all its lanes keeps one reference on it
     * (HINT_PINNED) */
    __device__ __forceinline__ uint32_t drop_stale(unsigned m, bool pin = false) {
        const bool stale = holds() && !ready();
        uint32_t hint = 0; /* the dropped frame + 1 (drop-behind policy) */
        if (__any_sync(m, stale)) {
            const uint64_t off = foff();
            if (stale) hint = (uint32_t)((((fb & XL_ADDR) - (uint64_t)r->pool) >> lg) + 1);
            if (pin && (r->prot & REGION_DROP_BEHIND)) {
                if (detail::unlink_lanes_pin(m, stale, r, page)) hint |= HINT_PINNED;
            } else {
                detail::unlink_lanes(m, stale, r, page);
            }
            if (stale) {
                x = off;
                fb = XL_VALID;
            }
        }
        return hint;
    }
    /* make every lane of m linked at its current offset */
    __device__ __forceinline__ void relink(unsigned m) {
        const uint64_t left = page;
        AP_FP_T(tr0);
        const uint32_t hint = drop_stale(m, true);
        AP_FP_T(tr1);
        AP_FP_ADD(m, 8, tr1 - tr0);
        uint32_t absent = 0;
        const bool minor_ok = !__any_sync(m, !holds()) || detail::try_link_minor<T, true>(m, x, page, r, lg, &absent);
        AP_FP_T(tr2);
        AP_FP_ADD(m, 9, tr2 - tr1);
        AP_FP_ADD(m, 10, 1);
        if (minor_ok) unpin(m, hint, left);
        if (!minor_ok) {
            /* bit 30: the caller reads the page itself (no value needed) */
            const detail::slow_out<T> o =
                detail::deref_slow<T>(m, x, page, r, hint | detail::absent_hint(absent) | (1u << 30), left);
            x = o.x;
            page = o.page;
        }
        sync_fb();
    }
    /* Forget the link without touching the count (it moved elsewhere). */
    __device__ __forceinline__ void detach() {
        x = foff();
        fb = XL_VALID;
    }
};

/* A GPU-scope acq_rel fence (see ptr::release_fenced, ptr::link_finish). */
__device__ __forceinline__ void fence_acq_rel() { detail::fence_gpu(); }

/* gvmmap (M17): an unlinked apointer to byte offset
 * `foff` of region `region` of the cache.  Read-only mappings only. */
template <class T>
__device__ __forceinline__ ptr<T> gvmmap(const dev_cache* c, uint32_t region, uint64_t foff) {
    return ptr<T>(c->regions + region, c->log2_page, foff);
}

}  // namespace ap

#endif /* AP_APOINTER_CUH_ */
