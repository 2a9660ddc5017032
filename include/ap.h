/*
 * ap.h — C ABI of the B200 apointer library (libapointer.so).
 *
 * ActivePointers (Shahar, Bergman, Silberstein, ISCA'16): a file mapped into
 * GPU memory is read through "active pointers" that translate file offsets in
 * software, cache the translation in a register, and take page faults that
 * are handled on the GPU (PAPER.md:9-13 abstract; §III, §IV).  This header is
 * the host-side boundary: create a page cache in HBM, map a "file" that lives
 * in pinned host memory, run the paper's microbenchmarks and its photo
 * collage, read statistics.  The device-side pointer type is in
 * include/ap/apointer.cuh.
 *
 * Conventions (every function):
 *   - returns int: AP_OK (0) on success, a negative AP_E* code on failure;
 *   - never throws, never aborts, writes results through out-parameters only
 *     on success;
 *   - pointers named *_dev are device pointers (cudaMalloc / torch CUDA
 *     tensors) owned by the caller; *_host are ordinary host pointers owned by
 *     the caller; the library never frees caller memory;
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream); asynchronous calls enqueue on it and return immediately;
 *   - a cache is bound to one device; calls switch to that device and
 *     restore the caller's current device before returning;
 *   - calls on one cache are not thread-safe against each other.
 */
#ifndef AP_H_
#define AP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------------------------------------------------------- errors */
#define AP_OK 0
#define AP_EINVAL (-1)    /* bad argument                                   */
#define AP_ENOMEM (-2)    /* device or pinned-host allocation failed         */
#define AP_ECUDA (-3)     /* a CUDA runtime call failed                      */
#define AP_EBUSY (-4)     /* live references / mapped regions prevent it     */
#define AP_ERANGE (-5)    /* region id / size / offset outside the layout    */
#define AP_EFAULT (-6)    /* device: dereference past the region or misaligned */
#define AP_ENOFRAME (-7)  /* device: no evictable frame (all pinned)         */
#define AP_ETIMEDOUT (-8) /* device: fault-path watchdog expired             */
#define AP_EPERM (-9)     /* device: store through a read-only mapping       */

/* Human-readable text for an AP_* code (static storage, never NULL). */
const char* ap_strerror(int code);

/* ------------------------------------------------------------- the cache */
typedef struct ap_cache_s* ap_cache_t;
typedef uint32_t ap_region_t;

/* ap_cache_create — the GPU page cache (§V "page cache in
 * GPU memory"; frames of page_size bytes, PAPER.md:363 uses 4 KB).
 *   frames     number of page frames, 1 <= frames < 2^28
 *   page_size  bytes per page: a power of two in [4096, 2 MiB]
 *   device     CUDA device ordinal
 * Allocates frames*page_size bytes of HBM (page_size aligned), the frame
 * owner table (8 B/frame), the free-frame array (4 B/frame), statistics and
 * the region table.  Errors: AP_EINVAL (bad size), AP_ENOMEM (HBM),
 * AP_ECUDA. */
int ap_cache_create(uint64_t frames, uint32_t page_size, int device, ap_cache_t* out);

/* Frees everything. AP_EBUSY while regions are still mapped. */
int ap_cache_destroy(ap_cache_t cache);

/* ap_mmap — map a read-only "file" (PAPER.md:125, 131 gvmmap(size, O_RDONLY,
 * fd, foffset); the file lives in host RAM as in PAPER.md:367, 428).
 *   host_buf  the file bytes in host memory, 16-B aligned, caller-owned; it
 *             must stay valid and unmodified until ap_munmap.  If it is not
 *             already page-locked it is registered (cudaHostRegisterMapped |
 *             ReadOnly) here and unregistered by ap_munmap.
 *   bytes     file size, > 0 (a ragged last page is zero-padded in its frame)
 * Creates the region's page table: one 8-B PTE per page, all EMPTY.
 * Errors: AP_EINVAL (NULL, 0 bytes, misaligned), AP_ERANGE (65535 regions
 * mapped, or > 2^48 pages), AP_ENOMEM, AP_ECUDA. */
int ap_mmap(ap_cache_t cache, const void* host_buf, uint64_t bytes, ap_region_t* out);

/* ap_mmap_prot — as ap_mmap with protection bits (NEXT N3; PAPER.md:134
 * Fig. 3 writes `*ptr = 25` through an apointer; "rw").
 *   prot  AP_PROT_READ, optionally | AP_PROT_WRITE.  A writable mapping
 *         registers the host bytes without the read-only flag; stores mark
 *         pages DIRTY and dirty pages are written back to host_buf when they
 *         are evicted, by ap_msync, ap_munmap and ap_cache_reset.
 * Errors: as ap_mmap; AP_EINVAL for other prot bits. */
#define AP_PROT_READ 1
#define AP_PROT_WRITE 2
int ap_mmap_prot(ap_cache_t cache, const void* host_buf, uint64_t bytes, int prot,
                 ap_region_t* out);

/* ap_msync — write every dirty resident page of a writable region back to
 * its host bytes and mark it clean (synchronises; no kernel may be using the
 * region).  No-op for read-only regions. */
int ap_msync(ap_cache_t cache, ap_region_t region);

/* Unmap: frames holding the region's pages go back to the free list.
 * AP_EBUSY if any page of the region still has a positive reference count
 * (a linked apointer). */
int ap_munmap(ap_cache_t cache, ap_region_t region);

/* ------------------------------------------ peer page caches (NEXT N2)
 * SURVEY 8(f) N2; PAPER.md:33 names distributed shared memory across GPUs as
 * a motivation.  Several caches (typically one per GPU) may map the same
 * file.  Declaring another cache's region as a peer of `region` makes a
 * major fault first look the page up in the peer's page table and, if it is
 * resident there, copy the peer's frame (HBM-to-HBM over NVLink 5 / the same
 * HBM) instead of reading the page over the host link; the peer's page is
 * pinned by its reference count during the copy, so the peer
 * can keep running and evicting.  Both mappings must be read-only, have the
 * same size and the same page size.  Up to 7 peers per region, tried in the
 * order added.  The caller keeps every peer mapped (and its cache alive)
 * until ap_region_clear_peers (or ap_munmap) of `region` returns.
 * Errors: AP_EINVAL (mismatch, writable, peer == cache, GPUs without peer
 * access), AP_ERANGE (7 peers already), AP_ECUDA. */

/* Same process: `peer_region` of `peer` (any GPU with peer access to this
 * cache's GPU, or the same GPU). */
int ap_region_add_peer(ap_cache_t cache, ap_region_t region, ap_cache_t peer,
                       ap_region_t peer_region);

/* Across processes (one process per GPU): ap_region_export writes a plain
 * byte record (CUDA IPC handles of the region's page table and of the frame
 * pool, plus sizes) that another process passes to ap_region_add_peer_ipc,
 * e.g. after an all-gather over torch.distributed.  The exporting process
 * keeps the cache and region alive until the importers cleared their peers. */
typedef struct {
    uint8_t pte_handle[64];  /* cudaIpcMemHandle_t of the PTE array          */
    uint8_t pool_handle[64]; /* cudaIpcMemHandle_t of the frame pool block   */
    uint64_t pool_offset;    /* frame pool start inside that block           */
    uint64_t bytes;          /* region size                                  */
    uint32_t page_size;
    int32_t device;          /* exporter's device ordinal (informational)    */
} ap_peer_handle_t;
int ap_region_export(ap_cache_t cache, ap_region_t region, ap_peer_handle_t* out);
int ap_region_add_peer_ipc(ap_cache_t cache, ap_region_t region, const ap_peer_handle_t* h);

/* Forget every peer of `region` (and close the IPC mappings); synchronises. */
int ap_region_clear_peers(ap_cache_t cache, ap_region_t region);

/* Device-accessible alias of the region's host bytes (the zero-copy view the
 * fault path fills from). Useful for raw-pointer twins. */
int ap_region_devptr(ap_cache_t cache, ap_region_t region, const void** out);

/* ------------------------------------------------------------ statistics */
typedef struct {
    uint64_t major;       /* major faults = page fills            */
    uint64_t minor;       /* minor faults = links to a resident page              */
    uint64_t fill_bytes;  /* bytes read from host memory by fills                 */
    uint64_t evictions;   /* frames reclaimed from refcount-0 pages               */
    uint64_t waits;       /* fault rounds that had to back off                    */
    uint64_t downgrades;  /* lanes proactively unlinked under frame pressure      */
    uint64_t nofree;      /* allocation attempts that found no evictable frame    */
    uint64_t unlinks;     /* warp-aggregated refcount decrements (0 unless the    *
                           * library is built with -DAP_COUNT_UNLINKS)           */
    uint64_t peer_fills;  /* major faults served from a peer cache (N2)           */
    uint64_t peer_bytes;  /* bytes those fills copied from peer frames            */
    uint64_t backoff_spins;   /* = waits (SURVEY B5's name)                       */
    uint64_t live_refcnt_sum; /* sum of the reference counts in the page tables *
                               * now: 0 whenever no apointer is linked  */
    int64_t err;              /* the sticky device error word (AP_OK if none),  *
                               * read without clearing it                       */
} ap_stats_t;

/* Sum of the device counters since create/reset, the live reference count
 * and the sticky error word (synchronises the device). */
int ap_cache_stats(ap_cache_t cache, ap_stats_t* out);

/* Evict every page, rebuild the free list, zero the counters: the next run
 * starts cold ("clearing the GPU buffer cache between runs").
 * AP_EBUSY if any page has a positive reference count. Synchronises. */
int ap_cache_reset(ap_cache_t cache);

/* Victim-selection policy of the eviction path.
 *   AP_POLICY_CLOCK   second-chance clock over frames (default)
 *   AP_POLICY_RANDOM  random victims from `seed` (test-only: output must not
 *                     depend on eviction order)                         */
#define AP_POLICY_CLOCK 0
#define AP_POLICY_RANDOM 1
/*   AP_POLICY_SEQUENTIAL  the clock, plus drop-behind: a warp that faults
 *                     right after its pointer left a page first reuses that
 *                     page's frame when no other pointer holds it (a hint for
 *                     single-pass streams, like MADV_SEQUENTIAL; pages that
 *                     are read again are better served by the plain clock) */
#define AP_POLICY_SEQUENTIAL 2
int ap_cache_set_policy(ap_cache_t cache, int policy, uint64_t seed);

/* Fault-path tunables: max_claims = pages one warp claims per fault round
 * (1 = the paper's sequential handling); sweep_steps = clock
 * steps (32 frames each) before an allocation gives up and backs off;
 * timeout_ms = watchdog for one dereference (0 = default 20000; a new cache
 * takes its default from the environment variable AP_TIMEOUT_MS if set, a
 * diagnostics aid). */
int ap_cache_set_tuning(ap_cache_t cache, uint32_t max_claims, uint32_t sweep_steps,
                        uint32_t timeout_ms);

/* Back-off of a warp whose page is being loaded by another warp or that
 * found no evictable frame: __nanosleep from min_ns doubling to max_ns
 * (defaults 64 / 4096). */
int ap_cache_set_backoff(ap_cache_t cache, uint32_t min_ns, uint32_t max_ns);

/* Sticky device error word (AP_EFAULT / AP_ENOFRAME / AP_ETIMEDOUT), cleared
 * on read; AP_OK if none. Synchronises. */
int ap_last_device_error(ap_cache_t cache);

/* Debug dumps for the invariant checks (synchronise):
 *   owner_host[frames]  0 = none, else ((region+1) << 48) | page
 *   free_left           frames still on the free list
 *   pte_host[npages]    bits 63:62 state (0 EMPTY, 1 LOADING, 2 VALID),
 *                       61 reference bit, 60 dirty, 59:32 frame,
 *                       31:0 reference count */
int ap_cache_dump(ap_cache_t cache, uint64_t* owner_host, uint64_t* free_left);
int ap_region_npages(ap_cache_t cache, ap_region_t region, uint64_t* npages);
int ap_region_dump_pte(ap_cache_t cache, ap_region_t region, uint64_t* pte_host);

/* Fault pages [first_page, first_page+npages) of a region into the cache
 * (one warp per page dereferences it through an apointer); they stay
 * resident with reference count 0. Asynchronous on `stream`. */
int ap_prefill(ap_cache_t cache, ap_region_t region, uint64_t first_page, uint64_t npages,
               void* stream);

/* ------------------------------------------------- microbenchmark (§VI-A/C) */
#define AP_SEQ 0       /* warp w reads units w, w+W, ... sequentially         */
#define AP_UNIFORM 1   /* uniform-random element offsets                      */
#define AP_DIVERGENT 2 /* the 32 lanes of a warp on 32 distinct pages         */
#define AP_SEQ_QUEUE 3 /* AP_SEQ's units, handed out in order from a device   *
                        * counter (the next free warp takes the next unit);    *
                        * out_copy and AP_ACCESS_TILE only                     */

#define AP_MODE_APOINTER 0 /* read through ap::ptr<T> (the method)           */
#define AP_MODE_RAW 1      /* identical kernel on a raw pointer (the twin,     *
                            * PAPER.md:304 "two versions of every benchmark") */

typedef struct {
    int32_t pattern;           /* AP_SEQ | AP_UNIFORM | AP_DIVERGENT | AP_SEQ_QUEUE */
    uint32_t elem_bytes;       /* 4, 8 or 16                                     */
    uint32_t grid, block;      /* launch shape; block a multiple of 32, <= 1024  */
    uint32_t reads_per_thread; /* UNIFORM / DIVERGENT                            */
    uint32_t passes;           /* SEQ: sweeps over [0, span)                     */
    uint32_t unit_bytes;       /* SEQ: bytes per warp unit (multiple of 32*elem, *
                                *      divides the page size)                    */
    uint32_t page_bytes;       /* DIVERGENT: page size of the pattern            */
    uint64_t span_bytes;       /* SEQ: bytes swept; UNIFORM: offsets drawn from [0, span_bytes); 0 = whole region */
    uint64_t seed;             /* UNIFORM / DIVERGENT offset generator seed       */
    int32_t mode;              /* AP_MODE_APOINTER | AP_MODE_RAW                 */
    int32_t out_copy;          /* SEQ: out receives the bytes read at their      *
                                * offsets (span bytes) instead of checksums      */
    const void* raw_base;      /* AP_MODE_RAW: device-readable file bytes (an HBM *
                                * copy, or ap_region_devptr for zero-copy)       */
    int32_t access;            /* SEQ, apointer mode: AP_ACCESS_TILE (default,    *
                                * one translation check per 8 accesses),         *
                                * AP_ACCESS_DEREF (`v = *q; q += 32` per access), *
                                * AP_ACCESS_RANGE (one check per unit, then plain *
                                * loads through the linked translation)          */
} ap_bench_cfg;

#define AP_ACCESS_TILE 0
#define AP_ACCESS_DEREF 1
#define AP_ACCESS_RANGE 2
#define AP_ACCESS_AHEAD 3 /* TILE + the next unit linked split-phase under the last tile */
#define AP_ACCESS_PAIR 4  /* TILE over two units whose links are issued together */
#define AP_ACCESS_TMA 5   /* 16-B checksums staged through shared memory by TMA bulk copies */

/* Run one microbenchmark launch (asynchronous on `stream`).
 * out_dev: uint64[grid*block] per-thread FNV-1a-64 checksums over the values
 * the thread read in access order, or
 * span bytes when out_copy.  Errors: AP_EINVAL (cfg), AP_ECUDA (launch). */
int ap_bench_read(ap_cache_t cache, ap_region_t region, const ap_bench_cfg* cfg, void* out_dev,
                  void* stream);

/* End-to-end variant: the same launch with the result copied into host
 * memory (out_host, caller-owned), synchronising; *seconds = wall time of
 * launch + device->host copy measured with CUDA events. */
int ap_bench_read_host(ap_cache_t cache, ap_region_t region, const ap_bench_cfg* cfg,
                       void* out_host, double* seconds);

/* ap_bench_write — stores through apointers into a writable region (NEXT
 * N3, Fig. 3 `*ptr = 25`).  cfg: pattern AP_SEQ (every element of
 * [0, span) once, warp units as ap_bench_read) or AP_UNIFORM (race-free
 * permutation: element (t*R+i)*a mod M, a = the odd number nearest below
 * 0.618*M coprime with M; needs grid*block*R <= M <= 2^32);
 * value at element e = low bytes of sm64(seed ^ e) (16-B: sm64(seed^2e),
 * sm64(seed^(2e+1))).  The host bytes change once the pages are written back
 * (eviction, ap_msync, ap_munmap).  Asynchronous on `stream`. */
int ap_bench_write(ap_cache_t cache, ap_region_t region, const ap_bench_cfg* cfg, void* stream);

/* ap_bench_copy — dst[e] = src[e] for the SEQ pattern of cfg, reading and
 * writing through apointers (the copy kernel of PAPER.md:310-316).  dst must
 * be writable.  cfg->mode = AP_MODE_RAW runs the raw twin (the same loop on
 * plain pointers): cfg->raw_base is a device buffer of 2 * span bytes, src =
 * its first half, dst = its second half (the regions are only validated).
 * Asynchronous on `stream`. */
int ap_bench_copy(ap_cache_t cache, ap_region_t src, ap_region_t dst, const ap_bench_cfg* cfg,
                  void* stream);

/* ap_bench_compute — the compute-intensity workloads of PAPER.md:332-359
 * (Fig. 6a/6b; NEXT N4), apointer version or raw twin (mode).
 *   work   0 ADD (acc += a[i] + b[i], b = a + span), 1 READ, 2 RANDOM-N (LCG
 *          x = x*1664525 + 1013904223 iterated `iters` times), 3 REDUCE (warp
 *          sum by shuffles), 4 FFT (32-point complex FFT across the warp,
 *          re/im = low/high 16 bits, acc += trunc(|X|^2 / 65536)), 5 BITONIC
 *          (warp bitonic sort, acc += sorted * (lane + 1));
 *   elem_bytes 4 or 16 (a 16-B load feeds four independent word lanes);
 *   span_bytes per vector, a multiple of the page size; warp w reads pages
 *          w, w+W, ... one 4/16-B access at a time (`*q; q += 32`);
 * out_dev: uint64[grid*block] per-thread accumulators.  Asynchronous. */
typedef struct {
    int32_t work;
    uint32_t elem_bytes;
    uint32_t grid, block;
    uint32_t iters;
    uint64_t span_bytes;
    int32_t mode;
    const void* raw_base;
} ap_compute_cfg;
int ap_bench_compute(ap_cache_t cache, ap_region_t region, const ap_compute_cfg* cfg,
                     uint64_t* out_dev, void* stream);

/* ap_bench_latency — Table I analogue: one warp, all
 * lanes on one (prefilled) page, coalesced 4-B accesses; op = 0 raw read,
 * 1 apointer read, 2 raw increment, 3 apointer increment, 4 raw read+inc,
 * 5 apointer read+inc.  cycles[0] = mean clock64 cycles per op after
 * subtracting cycles[1], the cost of an empty timing pair.  The raw pointer
 * reads the same frame the apointer is linked to.  Synchronises. */
int ap_bench_latency(ap_cache_t cache, ap_region_t region, int op, uint32_t reps,
                     uint64_t* cycles);

/* ---------------------------------------------------- photo collage (§VI-E) */
typedef struct {
    const uint8_t* target_dev;   /* W*H*3 uint8 RGB, interleaved, row-major       */
    uint32_t W, H;               /* multiples of 32                               */
    uint32_t L, K;               /* LSH tables, projections per table (K <= 16)   */
    uint32_t bucket_bits;        /* 1..30: buckets per table = 2^bucket_bits       */
    int32_t w;                   /* LSH bucket width, > 0                          */
    const int16_t* proj_dev;     /* [L][K][768]                                    */
    const int32_t* bias_dev;     /* [L][K]                                         */
    const uint32_t* offsets_dev; /* [L][2^bucket_bits + 1] bucket CSR offsets      */
    const uint32_t* ids_dev;     /* [L][N] record ids, ascending per bucket        */
    uint64_t N;                  /* records in the file                            */
    uint32_t rec_stride;         /* bytes between records (4096 = padded, 3072)   */
    uint32_t group;              /* candidates per warp iteration: 1, 2, 4, 8, 16  *
                                  * or 32 (32 / group lanes read each record)      */
    uint64_t block_begin;        /* first query block (row-major 32x32 blocks)     */
    uint64_t block_count;        /* number of query blocks                        */
    int32_t mode;                /* AP_MODE_APOINTER | AP_MODE_RAW                 */
    const void* raw_base;        /* AP_MODE_RAW: device-readable record file       */
    int32_t schedule;            /* AP_SCHED_NATURAL: CTA i = block i (the paper's *
                                  * single kernel); AP_SCHED_LSH: blocks are first *
                                  * sorted by their LSH keys (an extra key kernel  *
                                  * + radix sort) so blocks sharing buckets run    *
                                  * together and reuse cached records;           *
                                  * AP_SCHED_TABLE: the work unit is one block's  *
                                  * candidates from one table, units sorted by    *
                                  * (table, bucket), so every unit reading a      *
                                  * bucket runs together; the block's winner is   *
                                  * the atomic 64-bit min over its L units.       *
                                  * Results are identical (per-block argmin).     */
    /* AP_SCHED_TABLE only: run the slice [unit_begin, unit_begin + unit_count)
     * of the L * block_count units in (table, bucket) order (unit_count 0 =
     * all).  Blocks whose units are not all in the slice keep a partial
     * minimum or the sentinel: ranks that split the units combine their
     * winners with an unsigned 64-bit MIN reduction (multi-GPU, §8(e)). */
    uint64_t unit_begin;
    uint64_t unit_count;
    /* Record-id windows (AP_SCHED_TABLE / _MH only; 0 or 1 = off): the units
     * run id_chunks times, pass c reading only the candidates with record
     * id in [c*N/id_chunks, (c+1)*N/id_chunks).  A record is then needed in
     * one pass only, whichever tables list it, so with windows whose touched
     * records fit the cache it is filled about once (the LSH tables list it
     * up to L times).  The keys pass keeps every block's histogram and
     * bucket ranges in scratch (3 KiB + 8 B * L per block) for the passes.
     * Results are identical (the per-block minimum is an atomic min). */
    uint32_t id_chunks;
    /* Record-id range (per-table schedules only; id_end 0 = all records):
     * only candidates with id in [id_begin, id_end) are read; id_chunks then
     * splits this range.  Multi-GPU "by records": rank r takes the r-th
     * slice of the ids and runs every unit, so each GPU's page cache only
     * ever holds its own shard of the file; the partial winners are combined
     * with the same 64-bit MIN reduction as the bucket partition. */
    uint32_t id_begin;
    uint32_t id_end;
    /* AP_COLLAGE_ACCUMULATE: winners_dev is NOT initialised; every block's
     * result is folded into it with the 64-bit lexicographic (dist, idx) min
     * (R-A3), whatever the schedule, so partitions run by other calls, other
     * caches or other GPUs can accumulate into one winners array (initialise
     * it once with ap_winners_init).  AP_COLLAGE_SYSTEM: that min is a
     * system-scope atomic (winners_dev is another GPU's memory reached over
     * NVLink peer access, or a CUDA IPC mapping shared across processes).
     * 0 = the default: winners_dev is written from scratch. */
    uint32_t flags;
} ap_collage_in;

#define AP_COLLAGE_ACCUMULATE 1u
#define AP_COLLAGE_SYSTEM 2u

#define AP_SCHED_NATURAL 0
#define AP_SCHED_LSH 1
#define AP_SCHED_TABLE 2
/* AP_SCHED_TABLE_MH: AP_SCHED_TABLE units sorted by (MinHash of the unit's
 * bucket = its smallest record id, table, bucket): a bucket's units stay
 * together and buckets of different tables sharing records come close in
 * time.  bucket_bits <= 24.  unit_begin/unit_count slice this order. */
#define AP_SCHED_TABLE_MH 3

/* ap_collage_run — the collage kernel ("calculates the
 * histogram of each 32x32 block, computes its LSH keys, reads the candidate
 * histograms from the respective buckets stored in a file, exhaustively
 * searches for the closest ones among the candidates, and in the end produces
 * the indexes of the images"; all in one kernel).  Records are read through
 * apointers over `records` (mode APOINTER).  winners_dev: uint32
 * [block_count][2] = (image index, squared Euclidean distance); a block with
 * no candidate gets (0xFFFFFFFF, 0xFFFFFFFF).  Asynchronous on `stream`.
 * Errors: AP_EINVAL (W/H not multiples of 32, K > 16, group), AP_ECUDA. */
int ap_collage_run(ap_cache_t cache, ap_region_t records, const ap_collage_in* in,
                   uint32_t* winners_dev, void* stream);

/* ap_winners_init — set nblocks winners to the empty sentinel
 * (0xFFFFFFFF, 0xFFFFFFFF) (R-A4), the identity of the winners' min, before
 * partitions accumulate into them (AP_COLLAGE_ACCUMULATE).  Asynchronous. */
int ap_winners_init(uint32_t* winners_dev, uint64_t nblocks, void* stream);

/* ---------------------------------------- device buffers across processes
 * One process per GPU (the framework's launch model): a buffer of one
 * process's GPU is made addressable by the others with CUDA IPC, so their
 * kernels can combine results into it directly over NVLink (e.g. the
 * collage winners with AP_COLLAGE_ACCUMULATE | AP_COLLAGE_SYSTEM) -- no
 * collective in the data path.  ap_ipc_export works on any address inside a
 * cudaMalloc allocation of the current process; the handle is plain bytes
 * (send it with any host-side channel, e.g. torch.distributed's object
 * all-gather).  ap_ipc_import maps it on `device` and returns the same
 * address inside the mapping; ap_ipc_close unmaps (pass the address
 * ap_ipc_import returned).  The exporter keeps the buffer alive until every
 * importer closed it.  Errors: AP_EINVAL, AP_ECUDA. */
typedef struct {
    uint8_t handle[64]; /* cudaIpcMemHandle_t of the allocation            */
    uint64_t offset;    /* the exported address - the allocation's base    */
    uint64_t bytes;     /* bytes from the exported address to the end      */
    int32_t device;     /* exporter's device ordinal (informational)       */
    int32_t pid;        /* exporter's process id (informational)           */
} ap_ipc_handle_t;
int ap_ipc_export(const void* dev_ptr, ap_ipc_handle_t* out);
int ap_ipc_import(const ap_ipc_handle_t* h, int device, void** dev_ptr);
int ap_ipc_close(void* dev_ptr);

/* ---------------------------------------------- multi-GPU collage (§8(e))
 * One process drives G partitions of the collage, each on its own GPU with
 * its own page cache over the SAME pinned host file (read-only, so no
 * coherence is needed; the file is registered once for all of them).  The
 * query blocks are independent, so the partitions share
 * nothing but the winners: every partition's kernel folds its results
 * straight into the root GPU's winners array over NVLink peer memory
 * (system-scope 64-bit atomic min, AP_COLLAGE_ACCUMULATE | AP_COLLAGE_SYSTEM)
 * -- the combine is fused into the kernels' epilogue, no collective runs.
 * `devices` may repeat an ordinal: partitions sharing a GPU run concurrently
 * on their own streams (that is how a one-GPU box exercises G > 1). */
#define AP_MGPU_MAX 16
#define AP_PART_BLOCKS 0  /* contiguous block ranges (row bands)                  */
#define AP_PART_RECORDS 1 /* record-id slices: each cache holds one shard of the
                           * file; every partition runs all units (per-table
                           * schedules only)                                      */
#define AP_PART_UNITS 2   /* slices of the (table, bucket)-sorted units          */
typedef struct ap_mgpu_s* ap_mgpu_t;
typedef struct {
    const uint8_t* target_host;  /* W*H*3 uint8 RGB (caller-owned host memory)   */
    uint32_t W, H, L, K, bucket_bits;
    int32_t w;
    const int16_t* proj_host;    /* [L][K][768]                                  */
    const int32_t* bias_host;    /* [L][K]                                       */
    uint64_t N;
    uint32_t rec_stride, group;
    int32_t schedule;            /* AP_SCHED_*                                    */
    uint32_t id_chunks;          /* record-id windows per partition (0 = off)     */
    int32_t partition;           /* AP_PART_*                                     */
} ap_mgpu_collage_in;
typedef struct {
    double seconds;                   /* the step: CUDA events on the root from
                                       * before the first partition's launch to
                                       * after the last one's completion (winners
                                       * combined); cold caches, no host copies  */
    double part_seconds[AP_MGPU_MAX]; /* each partition's own kernels           */
    uint64_t fill_bytes[AP_MGPU_MAX]; /* host-link bytes filled per partition    */
    uint64_t major[AP_MGPU_MAX];
    int32_t device_error;             /* first sticky device error, or AP_OK     */
    int32_t nparts;
} ap_mgpu_report;

/* ap_mgpu_create — G = ngpu partitions on devices[0..G-1] (devices[0] is the
 * root holding the winners), each a page cache of frames_per_gpu frames of
 * page_size bytes mapping host_file (bytes, 16-B aligned, caller-owned,
 * valid until ap_mgpu_destroy).  Enables peer access from every partition's
 * GPU to the root.  Errors: AP_EINVAL (ngpu outside 1..AP_MGPU_MAX, no peer
 * access), AP_ENOMEM, AP_ECUDA. */
int ap_mgpu_create(int ngpu, const int* devices, const void* host_file, uint64_t bytes,
                   uint64_t frames_per_gpu, uint32_t page_size, ap_mgpu_t* out);
/* ap_mgpu_collage — one cold collage step over the G partitions: uploads the
 * target and LSH parameters and builds the bucket index on every GPU when
 * they differ from the previous call's (not timed), resets every cache, runs
 * the partitions concurrently, and copies the combined winners
 * uint32[blocks][2] into winners_host.  rep (optional) receives the timing
 * and per-partition counters.  Synchronises.  Errors: as ap_collage_run. */
int ap_mgpu_collage(ap_mgpu_t m, const ap_mgpu_collage_in* in, uint32_t* winners_host,
                    ap_mgpu_report* rep);
int ap_mgpu_destroy(ap_mgpu_t m);
/* One-shot convenience: create, one step, destroy. */
int ap_collage_mgpu(int ngpu, const int* devices, const void* host_file, uint64_t bytes,
                    uint64_t frames_per_gpu, uint32_t page_size, const ap_mgpu_collage_in* in,
                    uint32_t* winners_host, ap_mgpu_report* rep);

/* ap_lsh_build_index — the dataset index ("The dataset images
 * are placed in buckets indexed by the LSH keys derived from their
 * histograms").  Reads the N records of `records` (zero-copy from host
 * memory), computes each record's L keys, and writes per table the bucket
 * CSR: offsets_dev [L][2^bucket_bits+1], ids_dev [L][N] (ascending within a
 * bucket).  Synchronises `stream` before returning (it allocates scratch).
 * Errors: AP_EINVAL, AP_ENOMEM, AP_ECUDA. */
int ap_lsh_build_index(ap_cache_t cache, ap_region_t records, uint64_t N, uint32_t rec_stride,
                       uint32_t L, uint32_t K, uint32_t bucket_bits, int32_t w,
                       const int16_t* proj_dev, const int32_t* bias_dev, uint32_t* offsets_dev,
                       uint32_t* ids_dev, void* stream);

/* -------------------------------------------------------------- utilities */
/* Library version string and the compile target (static storage). */
const char* ap_version(void);

#ifdef __cplusplus
}
#endif
#endif /* AP_H_ */
