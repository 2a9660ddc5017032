/* ap_internal.cuh — host-side state of a cache, shared by the library's
 * translation units (runtime, benchmarks, collage).  Not installed. */
#ifndef AP_INTERNAL_CUH_
#define AP_INTERNAL_CUH_

#include <cuda_runtime.h>
#include <stdint.h>

#include <utility>
#include <vector>

#include "ap.h"
#include "ap/apointer.cuh"

constexpr uint32_t AP_MAX_REGIONS = 65535;

struct ap_region_host {
    const void* host_buf = nullptr; /* caller's pointer                      */
    const uint8_t* dev_alias = nullptr;
    uint64_t bytes = 0;
    uint64_t npages = 0;
    uint64_t* pte = nullptr; /* device                                     */
    const void* reg_base = nullptr; /* the library's host registration this
                                     * region holds a reference on, or null  */
    bool live = false;
    uint32_t prot = 1;       /* AP_PROT_*                                  */
    std::vector<ap::dev_peer> peers;  /* N2 peer caches (device-readable)  */
    ap::dev_peer* d_peers = nullptr;  /* their device copy                 */
    std::vector<void*> ipc_opened;    /* CUDA IPC mappings to close        */
    /* same-process peers: the regions this region copies from, and the
     * regions that copy from this one (its page table and frames must stay
     * alive while they do: ap_munmap answers AP_EBUSY) */
    std::vector<std::pair<struct ap_cache_s*, ap_region_t>> peer_src;
    std::vector<std::pair<struct ap_cache_s*, ap_region_t>> importers;
    bool exported = false; /* handed out with ap_region_export */
};

struct ap_cache_s {
    int device = 0;
    uint64_t frames = 0;
    uint32_t page = 0, log2_page = 0;
    void* pool_raw = nullptr;
    uint8_t* pool = nullptr;
    uint64_t* owner = nullptr;
    uint32_t* free_ids = nullptr;
    unsigned long long* free_head = nullptr;
    unsigned long long* clock_hand = nullptr;
    unsigned long long* seq_queue = nullptr; /* AP_SEQ_QUEUE unit counter */
    ap::dev_region* regions = nullptr;
    ap::dev_stats* stats = nullptr;
    int* err = nullptr;
    ap::dev_cache* d_cache = nullptr; /* device copy of `h` */
    ap::dev_cache h{};                /* host mirror         */
    std::vector<ap_region_host> reg;
    int num_sms = 148;
    uint64_t* slots = nullptr; /* -DAP_PT_HASH: the hash page table (N4 ablation) */
    uint32_t slot_bits = 0;
    uint64_t slot_keys = 0;    /* keys inserted at most (mapped pages + tombstones) */
    void* scratch = nullptr; /* grown on demand (collage schedule) */
    size_t scratch_bytes = 0;
};

/* Switch to the cache's device for the lifetime of the guard. */
struct ap_device_guard {
    int prev = -1;
    explicit ap_device_guard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) cudaSetDevice(dev);
    }
    ~ap_device_guard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

#define AP_CUDA_TRY(expr)                                  \
    do {                                                   \
        cudaError_t e__ = (expr);                          \
        if (e__ != cudaSuccess) {                          \
            ap_note_cuda_error(e__, #expr, __FILE__, __LINE__); \
            return AP_ECUDA;                               \
        }                                                  \
    } while (0)

void ap_note_cuda_error(cudaError_t e, const char* what, const char* file, int line);
/* Scratch device memory of at least `bytes` (synchronises only when it grows). */
void* ap_scratch(ap_cache_s* c, size_t bytes);
bool ap_region_ok(const ap_cache_s* c, ap_region_t r);

/* ap_sort.cu: stable LSD radix sort of n (key, value) pairs by the low
 * `bits` bits of the key (8-bit digits).  The passes ping-pong between
 * (keys, vals) and (keys_alt, vals_alt); *in_alt tells where the result
 * is.  scratch: ap_sort_scratch_bytes(n) bytes of device memory.
 * Asynchronous on s. */
size_t ap_sort_scratch_bytes(uint64_t n);
template <class K>
int ap_sort_pairs(K* keys, K* keys_alt, uint32_t* vals, uint32_t* vals_alt, uint64_t n, int bits,
                  void* scratch, cudaStream_t s, bool* in_alt);

#endif
