/*
 * ap_runtime.cu — host runtime of the apointer library: the page cache
 * (§V), file mapping (gvmmap, PAPER.md:125/131/367),
 * statistics, reset, dumps, prefill.  C ABI in include/ap.h.
 */
#include <cuda_runtime.h>
#include <cstddef>
#include <cstring>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <mutex>
#include <vector>

#include "ap_internal.cuh"

void ap_note_cuda_error(cudaError_t e, const char* what, const char* file, int line) {
    if (getenv("AP_VERBOSE"))
        fprintf(stderr, "[ap] %s:%d: %s -> %s\n", file, line, what, cudaGetErrorString(e));
}

extern "C" const char* ap_strerror(int code) {
    switch (code) {
        case AP_OK: return "ok";
        case AP_EINVAL: return "invalid argument";
        case AP_ENOMEM: return "out of memory";
        case AP_ECUDA: return "CUDA runtime error";
        case AP_EBUSY: return "busy: live references or mapped regions";
        case AP_ERANGE: return "out of range";
        case AP_EFAULT: return "device: dereference outside the mapped region or misaligned";
        case AP_ENOFRAME: return "device: no evictable frame";
        case AP_ETIMEDOUT: return "device: fault-path watchdog expired";
        case AP_EPERM: return "device: store through a read-only mapping";
        default: return "unknown error";
    }
}

extern "C" const char* ap_version(void) {
#ifdef AP_PT_HASH
    return "apointer-b200 0.1 (sm_100a; long apointer, no TLB, clock eviction; "
           "hash-table page table)";
#else
    return "apointer-b200 0.1 (sm_100a; long apointer, no TLB, clock eviction; dense page table)";
#endif
}

void* ap_scratch(ap_cache_s* c, size_t bytes) {
    if (c->scratch_bytes >= bytes) return c->scratch;
    cudaDeviceSynchronize();
    cudaFree(c->scratch);
    c->scratch = nullptr;
    c->scratch_bytes = 0;
    if (cudaMalloc(&c->scratch, bytes) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    c->scratch_bytes = bytes;
    return c->scratch;
}

bool ap_region_ok(const ap_cache_s* c, ap_region_t r) {
    return c && r < c->reg.size() && c->reg[r].live;
}

/* the device copy of a region's prot: + REGION_DROP_BEHIND under
 * AP_POLICY_SEQUENTIAL (read by a pointer's unlink when it leaves a page) */
static uint32_t region_prot_flags(const ap_cache_s* c, uint32_t prot) {
    return prot | (c->h.policy == ap::POLICY_SEQUENTIAL ? ap::REGION_DROP_BEHIND : 0u);
}

static int push_descriptor(ap_cache_s* c) {
    AP_CUDA_TRY(cudaMemcpy(c->d_cache, &c->h, sizeof(ap::dev_cache), cudaMemcpyHostToDevice));
    return AP_OK;
}

/* ------------------------------------------------------------ kernels */
__global__ void k_iota(uint32_t* a, uint64_t n) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x)
        a[i] = (uint32_t)i;
}

/* flag bit0: a positive reference count; bit1: an entry left LOADING. */
__global__ void k_scan_pte(const uint64_t* pte, uint64_t n, int* flag) {
    int f = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t e = pte[i];
        if (e & ap::PTE_RC_MASK) f |= 1;
        if ((e >> 62) == 1) f |= 2;
    }
    if (f) atomicOr(flag, f);
}

/* sum of the reference-count fields of n entries `stride` words apart
 * (B5's live_refcnt_sum) */
__global__ void k_refsum(const uint64_t* pte, uint64_t n, uint64_t stride,
                         unsigned long long* sum) {
    unsigned long long t = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x)
        t += pte[i * stride] & ap::PTE_RC_MASK;
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
    if ((threadIdx.x & 31) == 0 && t) atomicAdd(sum, t);
}

#ifdef AP_PT_HASH
/* hash page table (N4 ablation): per-slot scans of one region's keys */
__global__ void k_scan_slots(const uint64_t* slots, uint64_t n, uint64_t tag, int* flag) {
    int f = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        if ((slots[2 * i] >> 48) != tag || slots[2 * i] == ap::detail::PT_TOMB) continue;
        const uint64_t e = slots[2 * i + 1];
        if (e & ap::PTE_RC_MASK) f |= 1;
        if ((e >> 62) == 1) f |= 2;
    }
    if (f) atomicOr(flag, f);
}
__global__ void k_tomb_slots(uint64_t* slots, uint64_t n, uint64_t tag) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x)
        if ((slots[2 * i] >> 48) == tag && slots[2 * i] != ap::detail::PT_TOMB) {
            slots[2 * i] = ap::detail::PT_TOMB;
            slots[2 * i + 1] = 0;
        }
}
__global__ void k_dump_slots(const uint64_t* slots, uint64_t n, uint64_t tag, uint64_t* dense,
                             uint64_t npages) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t k = slots[2 * i];
        if ((k >> 48) == tag && k != ap::detail::PT_TOMB && (k & ap::PAGE_MASK48) < npages)
            dense[k & ap::PAGE_MASK48] = slots[2 * i + 1];
    }
}
#endif

__global__ void k_drop_owner(uint64_t* owner, uint64_t frames, uint64_t tag) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < frames;
         i += (uint64_t)gridDim.x * blockDim.x)
        if ((owner[i] >> 48) == tag) owner[i] = 0;
}

/* One warp per page: an apointer dereference faults it in; the pointer is
 * destroyed at scope exit, leaving the page resident with count 0. */
__global__ void k_prefill(const ap::dev_cache* __restrict__ c, uint32_t region, uint64_t first,
                          uint64_t npages) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) / 32;
    const uint64_t nwarps = (uint64_t)gridDim.x * blockDim.x / 32;
    const uint32_t lg = c->log2_page;
    for (uint64_t p = first + warp; p < first + npages; p += nwarps) {
        ap::ptr<uint32_t> q = ap::gvmmap<uint32_t>(c, region, p << lg);
        volatile uint32_t v = *q;
        (void)v;
    }
}

/* msync: one warp per page; VALID + DIRTY pages are copied back to the
 * file and marked clean (no kernel may run concurrently). */
__global__ void k_writeback(const ap::dev_cache* __restrict__ c, uint32_t region) {
    const ap::dev_region* r = c->regions + region;
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) / 32;
    const uint64_t nwarps = (uint64_t)gridDim.x * blockDim.x / 32;
    for (uint64_t p = warp; p < r->npages; p += nwarps) {
        uint64_t* q = AP_PTE_FIND(r, p);
#ifdef AP_PT_HASH
        if (!q) continue;
#endif
        const uint64_t e = *q;
        if ((e >> 62) == 2 && (e & ap::PTE_DIRTY)) {
            ap::detail::writeback_page(0xffffffffu, c, r, (e >> 32) & ap::PTE_FRAME_MASK, p);
            __syncwarp();
            if ((threadIdx.x & 31) == 0)
                atomicAnd((unsigned long long*)q, ~(unsigned long long)ap::PTE_DIRTY);
        }
    }
}

static int scan_refs(ap_cache_s* c, const ap_region_host& rg, int* result) {
    int* d_flag = nullptr;
    AP_CUDA_TRY(cudaMalloc(&d_flag, sizeof(int)));
    AP_CUDA_TRY(cudaMemset(d_flag, 0, sizeof(int)));
#ifdef AP_PT_HASH
    k_scan_slots<<<c->num_sms * 4, 256>>>(c->slots, 1ull << c->slot_bits,
                                          (uint64_t)(&rg - c->reg.data()) + 1, d_flag);
#else
    k_scan_pte<<<c->num_sms * 4, 256>>>(rg.pte, rg.npages, d_flag);
#endif
    int h = 0;
    cudaError_t e = cudaMemcpy(&h, d_flag, sizeof(int), cudaMemcpyDeviceToHost);
    cudaFree(d_flag);
    AP_CUDA_TRY(e);
    *result = h;
    return AP_OK;
}

/* Free list = every frame without an owner, ascending (R-A18). */
static int rebuild_free_list(ap_cache_s* c) {
    std::vector<uint64_t> owner(c->frames);
    AP_CUDA_TRY(cudaMemcpy(owner.data(), c->owner, c->frames * 8, cudaMemcpyDeviceToHost));
    std::vector<uint32_t> ids;
    ids.reserve(c->frames);
    for (uint64_t f = 0; f < c->frames; ++f)
        if (owner[f] == 0) ids.push_back((uint32_t)f);
    if (!ids.empty())
        AP_CUDA_TRY(cudaMemcpy(c->free_ids, ids.data(), ids.size() * 4, cudaMemcpyHostToDevice));
    AP_CUDA_TRY(cudaMemset(c->free_head, 0, sizeof(unsigned long long)));
    c->h.nfree = ids.size();
    return push_descriptor(c);
}

/* ------------------------------------------------------------ the cache */
extern "C" int ap_cache_create(uint64_t frames, uint32_t page_size, int device, ap_cache_t* out) {
    if (!out || frames == 0 || frames > ap::PTE_FRAME_MASK) return AP_EINVAL; /* < 2^28 */
    if (page_size < 4096 || page_size > (2u << 20) || (page_size & (page_size - 1))) return AP_EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return AP_EINVAL;
    ap_device_guard g(device);
    ap_cache_s* c = new ap_cache_s();
    c->device = device;
    c->frames = frames;
    c->page = page_size;
    c->log2_page = 0;
    while ((1u << c->log2_page) < page_size) ++c->log2_page;
    cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device);
    auto fail = [&](int code) {
        cudaFree(c->pool_raw);
        cudaFree(c->owner);
        cudaFree(c->free_ids);
        cudaFree(c->free_head);
        cudaFree(c->regions);
        cudaFree(c->stats);
        cudaFree(c->d_cache);
        delete c;
        cudaGetLastError();
        return code;
    };
    const uint64_t pool_bytes = frames * (uint64_t)page_size + page_size;
    if (cudaMalloc(&c->pool_raw, pool_bytes) != cudaSuccess) return fail(AP_ENOMEM);
    c->pool = (uint8_t*)(((uintptr_t)c->pool_raw + page_size - 1) & ~(uintptr_t)(page_size - 1));
    if (cudaMalloc(&c->owner, frames * 8) != cudaSuccess) return fail(AP_ENOMEM);
    if (cudaMalloc(&c->free_ids, frames * 4) != cudaSuccess) return fail(AP_ENOMEM);
    /* free_head, clock_hand and err share one small allocation */
    if (cudaMalloc(&c->free_head, 256) != cudaSuccess) return fail(AP_ENOMEM);
    c->clock_hand = c->free_head + 8;
    c->err = (int*)(c->free_head + 16);
    c->seq_queue = c->free_head + 24;
    if (cudaMalloc(&c->regions, sizeof(ap::dev_region) * AP_MAX_REGIONS) != cudaSuccess)
        return fail(AP_ENOMEM);
    if (cudaMalloc(&c->stats, sizeof(ap::dev_stats) * ap::STAT_SHARDS) != cudaSuccess)
        return fail(AP_ENOMEM);
    if (cudaMalloc(&c->d_cache, sizeof(ap::dev_cache)) != cudaSuccess) return fail(AP_ENOMEM);
#ifdef AP_PT_HASH
    /* 16x as many slots as frames */
    c->slot_bits = 10;
    while ((1ull << c->slot_bits) < 16 * frames) ++c->slot_bits;
    if (cudaMalloc(&c->slots, 16ull << c->slot_bits) != cudaSuccess ||
        cudaMemset(c->slots, 0, 16ull << c->slot_bits) != cudaSuccess)
        return fail(AP_ENOMEM);
#endif
    if (cudaMemset(c->owner, 0, frames * 8) != cudaSuccess ||
        cudaMemset(c->free_head, 0, 256) != cudaSuccess ||
        cudaMemset(c->regions, 0, sizeof(ap::dev_region) * AP_MAX_REGIONS) != cudaSuccess ||
        cudaMemset(c->stats, 0, sizeof(ap::dev_stats) * ap::STAT_SHARDS) != cudaSuccess)
        return fail(AP_ECUDA);
    k_iota<<<c->num_sms, 256>>>(c->free_ids, frames);
    if (cudaGetLastError() != cudaSuccess) return fail(AP_ECUDA);
    c->h.pool = c->pool;
    c->h.owner = c->owner;
    c->h.free_ids = c->free_ids;
    c->h.free_head = c->free_head;
    c->h.clock_hand = c->clock_hand;
    c->h.regions = c->regions;
    c->h.stats = c->stats;
    c->h.err = c->err;
    c->h.frames = frames;
    c->h.nfree = frames;
    c->h.policy_seed = 0;
    c->h.timeout_ns = 20000ull * 1000000ull;
    /* AP_TIMEOUT_MS (environment, diagnostics): a shorter fault-path
     * watchdog for every cache of the process, so a wait that cannot end
     * reports ERR_TIMEDOUT in seconds instead of tens of seconds */
    if (const char* e = getenv("AP_TIMEOUT_MS")) {
        const unsigned long long ms = strtoull(e, nullptr, 10);
        if (ms) c->h.timeout_ns = ms * 1000000ull;
    }
    c->h.log2_page = c->log2_page;
    c->h.policy = ap::POLICY_CLOCK;
    c->h.max_claims = 1;
    c->h.sweep_steps = 64;
    c->h.backoff_min_ns = 64;
    c->h.backoff_max_ns = 4096;
    if (push_descriptor(c) != AP_OK) return fail(AP_ECUDA);
    if (cudaDeviceSynchronize() != cudaSuccess) return fail(AP_ECUDA);
    *out = c;
    return AP_OK;
}

extern "C" int ap_cache_destroy(ap_cache_t c) {
    if (!c) return AP_EINVAL;
    for (auto& r : c->reg)
        if (r.live) return AP_EBUSY;
    ap_device_guard g(c->device);
    cudaDeviceSynchronize();
    cudaFree(c->pool_raw);
    cudaFree(c->owner);
    cudaFree(c->free_ids);
    cudaFree(c->free_head);
    cudaFree(c->regions);
    cudaFree(c->stats);
    cudaFree(c->d_cache);
    cudaFree(c->scratch);
    cudaFree(c->slots);
    delete c;
    return AP_OK;
}

/* ------------------------------------------------------------ regions */
/* Host registrations the library made, shared by every cache of the process
 * (several caches -- one per GPU -- map the same file): a registration is
 * undone only when the last region using it is unmapped.  Registrations the
 * caller made (cudaHostRegister / cudaHostAlloc / torch pin_memory) are used
 * as they are and never undone here. */
namespace {
struct host_reg {
    const uint8_t* base;
    uint64_t bytes;
    int refs;
    bool readonly;
};
std::mutex g_reg_mu;
std::vector<host_reg> g_regs;

host_reg* find_reg(const void* p, uint64_t bytes) {
    const uint8_t* b = (const uint8_t*)p;
    for (auto& r : g_regs)
        if (b >= r.base && b + bytes <= r.base + r.bytes) return &r;
    return nullptr;
}
}  // namespace

static void release_host_reg(const void* base) {
    std::lock_guard<std::mutex> lk(g_reg_mu);
    for (size_t i = 0; i < g_regs.size(); ++i)
        if (g_regs[i].base == (const uint8_t*)base) {
            if (--g_regs[i].refs == 0) {
                cudaHostUnregister(const_cast<uint8_t*>(g_regs[i].base));
                cudaGetLastError();
                g_regs.erase(g_regs.begin() + i);
            }
            return;
        }
}
extern "C" int ap_mmap(ap_cache_t c, const void* host_buf, uint64_t bytes, ap_region_t* out) {
    return ap_mmap_prot(c, host_buf, bytes, AP_PROT_READ, out);
}

extern "C" int ap_mmap_prot(ap_cache_t c, const void* host_buf, uint64_t bytes, int prot,
                            ap_region_t* out) {
    if (!c || !host_buf || bytes == 0 || !out) return AP_EINVAL;
    if (!(prot & AP_PROT_READ) || (prot & ~(AP_PROT_READ | AP_PROT_WRITE))) return AP_EINVAL;
#ifdef AP_PT_HASH
    if (prot & AP_PROT_WRITE) return AP_EINVAL; /* the N4 ablation maps read-only files */
#endif
    if (((uintptr_t)host_buf) & 15) return AP_EINVAL;
    const uint64_t npages = (bytes + c->page - 1) >> c->log2_page;
    if (npages >= (1ull << 48) || bytes >= (1ull << 60)) return AP_ERANGE;
    uint32_t id = 0;
    while (id < c->reg.size() && c->reg[id].live) ++id;
    if (id >= AP_MAX_REGIONS) return AP_ERANGE;
    ap_device_guard g(c->device);
    ap_region_host rg;
    rg.host_buf = host_buf;
    rg.bytes = bytes;
    rg.npages = npages;
    {
        std::lock_guard<std::mutex> lk(g_reg_mu);
        host_reg* hr = find_reg(host_buf, bytes);
        if (hr) {
            /* a registration this library made for another region/cache:
             * share it (a writable mapping cannot use a read-only one) */
            if ((prot & AP_PROT_WRITE) && hr->readonly) return AP_EINVAL;
            void* dp = nullptr;
            if (cudaHostGetDevicePointer(&dp, const_cast<void*>(host_buf), 0) != cudaSuccess) {
                cudaGetLastError();
                return AP_ECUDA;
            }
            rg.dev_alias = (const uint8_t*)dp;
            rg.reg_base = hr->base;
            ++hr->refs;
        }
    }
    if (!rg.dev_alias) {
        cudaPointerAttributes attr{};
        cudaError_t e = cudaPointerGetAttributes(&attr, host_buf);
        cudaGetLastError();
        if (e == cudaSuccess && attr.type == cudaMemoryTypeHost && attr.devicePointer) {
            /* pinned and mapped by the caller: used as is, never unregistered */
            rg.dev_alias = (const uint8_t*)attr.devicePointer;
        } else if (e == cudaSuccess && attr.type == cudaMemoryTypeDevice) {
            return AP_EINVAL; /* the backing store is host memory */
        } else {
            unsigned flags = cudaHostRegisterMapped | cudaHostRegisterPortable;
            int ro = 0;
            if (!(prot & AP_PROT_WRITE))
                cudaDeviceGetAttribute(&ro, cudaDevAttrHostRegisterReadOnlySupported, c->device);
            if (ro) flags |= cudaHostRegisterReadOnly;
            e = cudaHostRegister(const_cast<void*>(host_buf), bytes, flags);
            if (e != cudaSuccess && ro) {
                cudaGetLastError();
                ro = 0;
                e = cudaHostRegister(const_cast<void*>(host_buf), bytes,
                                     cudaHostRegisterMapped | cudaHostRegisterPortable);
            }
            if (e != cudaSuccess) {
                cudaGetLastError();
                return AP_ENOMEM;
            }
            void* dp = nullptr;
            if (cudaHostGetDevicePointer(&dp, const_cast<void*>(host_buf), 0) != cudaSuccess) {
                cudaHostUnregister(const_cast<void*>(host_buf));
                cudaGetLastError();
                return AP_ECUDA;
            }
            rg.dev_alias = (const uint8_t*)dp;
            rg.reg_base = host_buf;
            std::lock_guard<std::mutex> lk(g_reg_mu);
            g_regs.push_back(host_reg{(const uint8_t*)host_buf, bytes, 1, ro != 0});
        }
    }
    /* every failure below releases the registration reference taken above */
    auto fail = [&](int code) {
        if (rg.pte) cudaFree(rg.pte);
        if (rg.reg_base) release_host_reg(rg.reg_base);
        cudaGetLastError();
        return code;
    };
    if (cudaMalloc(&rg.pte, npages * 8) != cudaSuccess) {
        rg.pte = nullptr;
        return fail(AP_ENOMEM);
    }
    if (cudaMemset(rg.pte, 0, npages * 8) != cudaSuccess) return fail(AP_ECUDA);
#ifdef AP_PT_HASH
    if (2 * (c->slot_keys + npages) > (1ull << c->slot_bits)) {
        /* grow the table to >= 2x the keys: dirty pages go back to their
         * files, every page is evicted (a reset, which checks the live
         * table for references first), then the regions move to a fresh
         * table; the old keys and tombstones are gone, so the key count
         * restarts from the mapped pages */
        for (uint32_t i = 0; i < c->reg.size(); ++i)
            if (c->reg[i].live && (c->reg[i].prot & AP_PROT_WRITE)) {
                int rcw = ap_msync(c, i);
                if (rcw) return fail(rcw);
            }
        int rcr = ap_cache_reset(c);
        if (rcr) return fail(rcr);
        uint64_t live_pages = 0;
        for (uint32_t i = 0; i < c->reg.size(); ++i)
            if (c->reg[i].live) live_pages += c->reg[i].npages;
        uint32_t bits = c->slot_bits;
        while ((1ull << bits) < 2 * (live_pages + npages)) ++bits;
        uint64_t* ns = nullptr;
        if (cudaMalloc(&ns, 16ull << bits) != cudaSuccess) return fail(AP_ENOMEM);
        if (cudaMemset(ns, 0, 16ull << bits) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) {
            cudaFree(ns);
            return fail(AP_ECUDA);
        }
        cudaFree(c->slots);
        c->slots = ns;
        c->slot_bits = bits;
        for (uint32_t i = 0; i < c->reg.size(); ++i)
            if (c->reg[i].live) {
                ap::dev_region od{};
                if (cudaMemcpy(&od, c->regions + i, sizeof od, cudaMemcpyDeviceToHost) != cudaSuccess)
                    return fail(AP_ECUDA);
                od.pte = c->slots;
                od.pad_ = c->slot_bits;
                if (cudaMemcpy(c->regions + i, &od, sizeof od, cudaMemcpyHostToDevice) != cudaSuccess)
                    return fail(AP_ECUDA);
            }
        c->slot_keys = live_pages;
    }
    c->slot_keys += npages;
#endif
    ap::dev_region d{};
    d.host = rg.dev_alias;
    d.bytes = bytes;
    d.npages = npages;
#ifdef AP_PT_HASH
    d.pte = c->slots;
    d.pad_ = c->slot_bits;
#else
    d.pte = rg.pte;
#endif
    d.cache = c->d_cache;
    d.pool = c->pool;
    d.stats = c->stats;
    d.prot = region_prot_flags(c, (uint32_t)prot);
    d.id = id;
    d.live = 1;
    if (cudaMemcpy(c->regions + id, &d, sizeof d, cudaMemcpyHostToDevice) != cudaSuccess)
        return fail(AP_ECUDA);
    rg.live = true;
    rg.prot = (uint32_t)prot;
    if (id == c->reg.size()) c->reg.push_back(rg);
    else c->reg[id] = rg;
    *out = id;
    return AP_OK;
}

extern "C" int ap_msync(ap_cache_t c, ap_region_t r) {
    if (!ap_region_ok(c, r)) return AP_EINVAL;
    if (!(c->reg[r].prot & AP_PROT_WRITE)) return AP_OK;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    k_writeback<<<c->num_sms * 4, 256>>>(c->d_cache, r);
    AP_CUDA_TRY(cudaGetLastError());
    AP_CUDA_TRY(cudaDeviceSynchronize());
    return AP_OK;
}

extern "C" int ap_munmap(ap_cache_t c, ap_region_t r) {
    if (!ap_region_ok(c, r)) return AP_EINVAL;
    /* another cache still copies from this region's frames (a same-process
     * peer, ap_region_add_peer): it must clear its peers first */
    if (!c->reg[r].importers.empty()) return AP_EBUSY;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    if (!c->reg[r].peers.empty() || c->reg[r].d_peers) {
        int rcp = ap_region_clear_peers(c, r);
        if (rcp) return rcp;
        cudaFree(c->reg[r].d_peers);
        c->reg[r].d_peers = nullptr;
    }
    if (c->reg[r].prot & AP_PROT_WRITE) {
        int rc0 = ap_msync(c, r);
        if (rc0) return rc0;
    }
    ap_region_host& rg = c->reg[r];
    int flag = 0;
    int rc = scan_refs(c, rg, &flag);
    if (rc) return rc;
    if (flag) return AP_EBUSY;
    k_drop_owner<<<c->num_sms * 4, 256>>>(c->owner, c->frames, (uint64_t)r + 1);
#ifdef AP_PT_HASH
    k_tomb_slots<<<c->num_sms * 4, 256>>>(c->slots, 1ull << c->slot_bits, (uint64_t)r + 1);
#endif
    AP_CUDA_TRY(cudaGetLastError());
    rc = rebuild_free_list(c);
    if (rc) return rc;
    AP_CUDA_TRY(cudaMemset(c->regions + r, 0, sizeof(ap::dev_region)));
    AP_CUDA_TRY(cudaDeviceSynchronize());
    cudaFree(rg.pte);
    if (rg.reg_base) release_host_reg(rg.reg_base);
    rg = ap_region_host{};
    return AP_OK;
}

/* ------------------------------------------------------------ N2 peers */
/* dev_region::shared: the fault path's claim / publish / eviction RMWs on
 * this region's PTEs use system scope once another cache pins its pages */
static int set_region_shared(ap_cache_s* c, ap_region_t r, uint32_t v) {
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    AP_CUDA_TRY(cudaMemcpy((uint8_t*)(c->regions + r) + offsetof(ap::dev_region, shared), &v,
                           sizeof v, cudaMemcpyHostToDevice));
    return AP_OK;
}

static int push_region_peers(ap_cache_s* c, ap_region_t r) {
    ap_region_host& rg = c->reg[r];
    if (!rg.d_peers && cudaMalloc(&rg.d_peers, sizeof(ap::dev_peer) * ap::MAX_PEERS) != cudaSuccess) {
        cudaGetLastError();
        return AP_ENOMEM;
    }
    if (!rg.peers.empty())
        AP_CUDA_TRY(cudaMemcpy(rg.d_peers, rg.peers.data(), sizeof(ap::dev_peer) * rg.peers.size(),
                               cudaMemcpyHostToDevice));
    ap::dev_region d{};
    AP_CUDA_TRY(cudaMemcpy(&d, c->regions + r, sizeof d, cudaMemcpyDeviceToHost));
    d.peers = rg.d_peers;
    d.npeers = (uint32_t)rg.peers.size();
    AP_CUDA_TRY(cudaMemcpy(c->regions + r, &d, sizeof d, cudaMemcpyHostToDevice));
    AP_CUDA_TRY(cudaDeviceSynchronize());
    return AP_OK;
}

static int peer_compatible(const ap_cache_s* c, ap_region_t r, uint32_t page, uint64_t bytes) {
    const ap_region_host& rg = c->reg[r];
    if (page != c->page || bytes != rg.bytes) return AP_EINVAL;
    if (rg.prot & AP_PROT_WRITE) return AP_EINVAL;
    if (rg.peers.size() >= ap::MAX_PEERS) return AP_ERANGE;
    return AP_OK;
}

extern "C" int ap_region_add_peer(ap_cache_t c, ap_region_t r, ap_cache_t pc, ap_region_t pr) {
#ifdef AP_PT_HASH
    return AP_EINVAL; /* peers read a dense page table */
#endif
    if (!ap_region_ok(c, r) || !ap_region_ok(pc, pr) || c == pc) return AP_EINVAL;
    if (pc->reg[pr].prot & AP_PROT_WRITE) return AP_EINVAL;
    int rc = peer_compatible(c, r, pc->page, pc->reg[pr].bytes);
    if (rc) return rc;
    ap_device_guard g(c->device);
    if (pc->device != c->device) {
        int ok = 0;
        AP_CUDA_TRY(cudaDeviceCanAccessPeer(&ok, c->device, pc->device));
        if (!ok) return AP_EINVAL;
        cudaError_t e = cudaDeviceEnablePeerAccess(pc->device, 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
        else AP_CUDA_TRY(e);
    }
    AP_CUDA_TRY(cudaDeviceSynchronize());
    if (pc->reg[pr].importers.empty() && !pc->reg[pr].exported) {
        rc = set_region_shared(pc, pr, 1);
        if (rc) return rc;
    }
    c->reg[r].peers.push_back(ap::dev_peer{pc->reg[pr].pte, pc->pool});
    rc = push_region_peers(c, r);
    if (rc) {
        c->reg[r].peers.pop_back();
        return rc;
    }
    c->reg[r].peer_src.emplace_back(pc, pr);
    pc->reg[pr].importers.emplace_back(c, r);
    return AP_OK;
}

extern "C" int ap_region_export(ap_cache_t c, ap_region_t r, ap_peer_handle_t* out) {
#ifdef AP_PT_HASH
    return AP_EINVAL; /* peers read a dense page table */
#endif
    if (!ap_region_ok(c, r) || !out) return AP_EINVAL;
    if (c->reg[r].prot & AP_PROT_WRITE) return AP_EINVAL;
    static_assert(sizeof(cudaIpcMemHandle_t) <= sizeof out->pte_handle, "IPC handle size");
    ap_device_guard g(c->device);
    ap_peer_handle_t h{};
    cudaIpcMemHandle_t a, b;
    AP_CUDA_TRY(cudaIpcGetMemHandle(&a, c->reg[r].pte));
    AP_CUDA_TRY(cudaIpcGetMemHandle(&b, c->pool_raw));
    memcpy(h.pte_handle, &a, sizeof a);
    memcpy(h.pool_handle, &b, sizeof b);
    h.pool_offset = (uint64_t)(c->pool - (uint8_t*)c->pool_raw);
    h.bytes = c->reg[r].bytes;
    h.page_size = c->page;
    h.device = c->device;
    if (!c->reg[r].exported && c->reg[r].importers.empty()) {
        int rc = set_region_shared(c, r, 1);
        if (rc) return rc;
    }
    c->reg[r].exported = true;
    *out = h;
    return AP_OK;
}

extern "C" int ap_region_add_peer_ipc(ap_cache_t c, ap_region_t r, const ap_peer_handle_t* h) {
#ifdef AP_PT_HASH
    return AP_EINVAL; /* peers read a dense page table */
#endif
    if (!ap_region_ok(c, r) || !h) return AP_EINVAL;
    int rc = peer_compatible(c, r, h->page_size, h->bytes);
    if (rc) return rc;
    ap_device_guard g(c->device);
    cudaIpcMemHandle_t a, b;
    memcpy(&a, h->pte_handle, sizeof a);
    memcpy(&b, h->pool_handle, sizeof b);
    void* pte = nullptr;
    void* pool = nullptr;
    AP_CUDA_TRY(cudaIpcOpenMemHandle(&pte, a, cudaIpcMemLazyEnablePeerAccess));
    cudaError_t e = cudaIpcOpenMemHandle(&pool, b, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
        cudaIpcCloseMemHandle(pte);
        AP_CUDA_TRY(e);
    }
    ap_region_host& rg = c->reg[r];
    rg.ipc_opened.push_back(pte);
    rg.ipc_opened.push_back(pool);
    rg.peers.push_back(ap::dev_peer{(uint64_t*)pte, (const uint8_t*)pool + h->pool_offset});
    return push_region_peers(c, r);
}

extern "C" int ap_region_clear_peers(ap_cache_t c, ap_region_t r) {
    if (!ap_region_ok(c, r)) return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    ap_region_host& rg = c->reg[r];
    rg.peers.clear();
    if (rg.d_peers) {
        int rc = push_region_peers(c, r);
        if (rc) return rc;
    }
    for (void* p : rg.ipc_opened) cudaIpcCloseMemHandle(p);
    rg.ipc_opened.clear();
    /* the same-process peers no longer have this importer */
    for (auto& src : rg.peer_src) {
        auto& imp = src.first->reg[src.second].importers;
        for (size_t i = 0; i < imp.size(); ++i)
            if (imp[i].first == c && imp[i].second == r) {
                imp.erase(imp.begin() + i);
                break;
            }
    }
    rg.peer_src.clear();
    return AP_OK;
}

extern "C" int ap_region_devptr(ap_cache_t c, ap_region_t r, const void** out) {
    if (!ap_region_ok(c, r) || !out) return AP_EINVAL;
    *out = c->reg[r].dev_alias;
    return AP_OK;
}

extern "C" int ap_region_npages(ap_cache_t c, ap_region_t r, uint64_t* npages) {
    if (!ap_region_ok(c, r) || !npages) return AP_EINVAL;
    *npages = c->reg[r].npages;
    return AP_OK;
}

/* ------------------------------------------------------------ stats etc. */
extern "C" int ap_cache_stats(ap_cache_t c, ap_stats_t* out) {
    if (!c || !out) return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    std::vector<ap::dev_stats> s(ap::STAT_SHARDS);
    AP_CUDA_TRY(cudaMemcpy(s.data(), c->stats, sizeof(ap::dev_stats) * ap::STAT_SHARDS,
                           cudaMemcpyDeviceToHost));
    ap_stats_t t{};
    for (auto& x : s) {
        t.major += x.major;
        t.minor += x.minor;
        t.fill_bytes += x.fill_bytes;
        t.evictions += x.evictions;
        t.waits += x.waits;
        t.downgrades += x.downgrades;
        t.nofree += x.nofree;
        t.unlinks += x.unlinks;
        t.peer_fills += x.peer_fills;
        t.peer_bytes += x.peer_bytes;
    }
    t.backoff_spins = t.waits;
    /* live references: the count fields of every page-table entry */
    unsigned long long* d_sum = nullptr;
    AP_CUDA_TRY(cudaMalloc(&d_sum, sizeof(unsigned long long)));
    cudaError_t e = cudaMemset(d_sum, 0, sizeof(unsigned long long));
#ifdef AP_PT_HASH
    if (e == cudaSuccess) k_refsum<<<c->num_sms * 4, 256>>>(c->slots + 1, 1ull << c->slot_bits, 2, d_sum);
#else
    for (auto& rg : c->reg)
        if (e == cudaSuccess && rg.live) k_refsum<<<c->num_sms * 4, 256>>>(rg.pte, rg.npages, 1, d_sum);
#endif
    if (e == cudaSuccess) e = cudaGetLastError();
    unsigned long long sum = 0;
    if (e == cudaSuccess) e = cudaMemcpy(&sum, d_sum, sizeof sum, cudaMemcpyDeviceToHost);
    cudaFree(d_sum);
    AP_CUDA_TRY(e);
    t.live_refcnt_sum = sum;
    int err = 0; /* the sticky error word, not cleared (ap_last_device_error clears it) */
    AP_CUDA_TRY(cudaMemcpy(&err, c->err, sizeof(int), cudaMemcpyDeviceToHost));
    t.err = err;
    *out = t;
    return AP_OK;
}

extern "C" int ap_cache_reset(ap_cache_t c) {
    if (!c) return AP_EINVAL;
    /* caches that copy from this one (same-process peers) may have kernels
     * in flight on other GPUs pinning our frames: let them finish first */
    for (auto& rg : c->reg)
        for (auto& imp : rg.importers) {
            ap_device_guard gi(imp.first->device);
            AP_CUDA_TRY(cudaDeviceSynchronize());
        }
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    for (auto& rg : c->reg) {
        if (!rg.live) continue;
        int flag = 0;
        int rc = scan_refs(c, rg, &flag);
        if (rc) return rc;
        if (flag) return AP_EBUSY;
    }
    for (uint32_t i = 0; i < c->reg.size(); ++i)
        if (c->reg[i].live && (c->reg[i].prot & AP_PROT_WRITE)) {
            int rc = ap_msync(c, i); /* dirty pages reach the file before eviction */
            if (rc) return rc;
        }
    for (auto& rg : c->reg)
        if (rg.live) AP_CUDA_TRY(cudaMemset(rg.pte, 0, rg.npages * 8));
#ifdef AP_PT_HASH
    AP_CUDA_TRY(cudaMemset(c->slots, 0, 16ull << c->slot_bits));
    c->slot_keys = 0;
    for (auto& rg : c->reg)
        if (rg.live) c->slot_keys += rg.npages;
#endif
    AP_CUDA_TRY(cudaMemset(c->owner, 0, c->frames * 8));
    AP_CUDA_TRY(cudaMemset(c->free_head, 0, 256));
    AP_CUDA_TRY(cudaMemset(c->stats, 0, sizeof(ap::dev_stats) * ap::STAT_SHARDS));
    k_iota<<<c->num_sms, 256>>>(c->free_ids, c->frames);
    AP_CUDA_TRY(cudaGetLastError());
    c->h.nfree = c->frames;
    int rc = push_descriptor(c);
    if (rc) return rc;
    AP_CUDA_TRY(cudaDeviceSynchronize());
    return AP_OK;
}

extern "C" int ap_cache_set_policy(ap_cache_t c, int policy, uint64_t seed) {
    if (!c || (policy != AP_POLICY_CLOCK && policy != AP_POLICY_RANDOM &&
               policy != AP_POLICY_SEQUENTIAL))
        return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    c->h.policy = policy;
    c->h.policy_seed = seed;
    /* the regions' drop-behind flag follows the policy */
    for (uint32_t i = 0; i < c->reg.size(); ++i)
        if (c->reg[i].live) {
            const uint32_t prot = region_prot_flags(c, c->reg[i].prot);
            AP_CUDA_TRY(cudaMemcpy(&c->regions[i].prot, &prot, 4, cudaMemcpyHostToDevice));
        }
    return push_descriptor(c);
}

extern "C" int ap_cache_set_tuning(ap_cache_t c, uint32_t max_claims, uint32_t sweep_steps,
                                   uint32_t timeout_ms) {
    if (!c || max_claims == 0 || max_claims > 32 || sweep_steps == 0) return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    c->h.max_claims = max_claims;
    c->h.sweep_steps = sweep_steps;
    c->h.timeout_ns = (uint64_t)(timeout_ms ? timeout_ms : 20000) * 1000000ull;
    return push_descriptor(c);
}

extern "C" int ap_cache_set_backoff(ap_cache_t c, uint32_t min_ns, uint32_t max_ns) {
    if (!c || min_ns == 0 || max_ns < min_ns || max_ns > 1000000) return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    c->h.backoff_min_ns = min_ns;
    c->h.backoff_max_ns = max_ns;
    return push_descriptor(c);
}

extern "C" int ap_last_device_error(ap_cache_t c) {
    if (!c) return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    int e = 0;
    AP_CUDA_TRY(cudaMemcpy(&e, c->err, sizeof(int), cudaMemcpyDeviceToHost));
    AP_CUDA_TRY(cudaMemset(c->err, 0, sizeof(int)));
    return e;
}

extern "C" int ap_cache_dump(ap_cache_t c, uint64_t* owner_host, uint64_t* free_left) {
    if (!c || !owner_host || !free_left) return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
    AP_CUDA_TRY(cudaMemcpy(owner_host, c->owner, c->frames * 8, cudaMemcpyDeviceToHost));
    unsigned long long head = 0;
    AP_CUDA_TRY(cudaMemcpy(&head, c->free_head, 8, cudaMemcpyDeviceToHost));
    *free_left = head >= c->h.nfree ? 0 : c->h.nfree - head;
    return AP_OK;
}

extern "C" int ap_region_dump_pte(ap_cache_t c, ap_region_t r, uint64_t* pte_host) {
    if (!ap_region_ok(c, r) || !pte_host) return AP_EINVAL;
    ap_device_guard g(c->device);
    AP_CUDA_TRY(cudaDeviceSynchronize());
#ifdef AP_PT_HASH
    /* a dense view of the region's slots (EMPTY where the page has none) */
    uint64_t* dense = nullptr;
    AP_CUDA_TRY(cudaMalloc(&dense, c->reg[r].npages * 8));
    AP_CUDA_TRY(cudaMemset(dense, 0, c->reg[r].npages * 8));
    k_dump_slots<<<c->num_sms * 4, 256>>>(c->slots, 1ull << c->slot_bits, (uint64_t)r + 1, dense,
                                          c->reg[r].npages);
    cudaError_t e = cudaMemcpy(pte_host, dense, c->reg[r].npages * 8, cudaMemcpyDeviceToHost);
    cudaFree(dense);
    AP_CUDA_TRY(e);
#else
    AP_CUDA_TRY(cudaMemcpy(pte_host, c->reg[r].pte, c->reg[r].npages * 8, cudaMemcpyDeviceToHost));
#endif
    return AP_OK;
}

extern "C" int ap_prefill(ap_cache_t c, ap_region_t r, uint64_t first, uint64_t npages,
                          void* stream) {
    if (!ap_region_ok(c, r) || first + npages > c->reg[r].npages) return AP_EINVAL;
    if (npages == 0) return AP_OK;
    ap_device_guard g(c->device);
    const uint64_t warps = std::min<uint64_t>(npages, (uint64_t)c->num_sms * 32);
    const unsigned blocks = (unsigned)((warps * 32 + 255) / 256);
    k_prefill<<<blocks, 256, 0, (cudaStream_t)stream>>>(c->d_cache, r, first, npages);
    AP_CUDA_TRY(cudaGetLastError());
    return AP_OK;
}

#ifdef AP_FAULT_PROF
/* diagnostic builds only (AP_FAULT_PROF): the fault-path phase counters */
namespace ap {
namespace detail {
__device__ unsigned long long ap_fprof[16];
}
}  // namespace ap
extern "C" int ap_fault_prof(uint64_t* out16, int reset) {
    AP_CUDA_TRY(cudaDeviceSynchronize());
    AP_CUDA_TRY(cudaMemcpyFromSymbol(out16, ap::detail::ap_fprof, 16 * sizeof(uint64_t)));
    if (reset) {
        static const unsigned long long zero[16] = {};
        AP_CUDA_TRY(cudaMemcpyToSymbol(ap::detail::ap_fprof, zero, sizeof(zero)));
    }
    return AP_OK;
}
#endif
