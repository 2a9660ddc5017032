/*
 * ap_mgpu.cu — multi-GPU collage and the CUDA IPC
 * plumbing of the one-process-per-GPU path.  C ABI in include/ap.h.
 *
 * The collage's query blocks are independent (each 32x32 block
 * searches its own candidates), so G partitions run on G GPUs, each with its
 * own page cache over the same pinned host file (read-only: no coherence).
 * The only exchange is the per-block winner, and it needs no collective: the
 * collage kernel of every partition folds each block's result into the root
 * GPU's winners array with a system-scope 64-bit atomic min over NVLink peer
 * memory (ap_collage_in.flags = AP_COLLAGE_ACCUMULATE | AP_COLLAGE_SYSTEM),
 * tile by tile as blocks finish -- the combine is fused into the kernels'
 * epilogue and overlaps the other partitions' work.  With one process per
 * GPU the same fold reaches the root's array through a CUDA IPC mapping
 * (ap_ipc_export / ap_ipc_import).
 */
#include <cuda.h> /* types only: driver entry points are fetched at run time, so the
                     library loads (and its CPU tests run) without libcuda */
#include <cuda_runtime.h>
#include <string.h>
#include <unistd.h>

#include <vector>

#include "ap_internal.cuh"

/* ------------------------------------------------------------------ IPC */
/* base and size of the allocation holding p (cuMemGetAddressRange through
 * cudaGetDriverEntryPoint: no link-time dependency on libcuda) */
static int alloc_range(const void* p, CUdeviceptr* base, size_t* size) {
    typedef CUresult (*range_fn)(CUdeviceptr*, size_t*, CUdeviceptr);
    static range_fn fn = nullptr;
    if (!fn) {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) !=
                cudaSuccess || q != cudaDriverEntryPointSuccess || !f) {
            cudaGetLastError();
            return AP_ECUDA;
        }
        fn = (range_fn)f;
    }
    return fn(base, size, (CUdeviceptr)p) == CUDA_SUCCESS ? AP_OK : AP_EINVAL;
}

extern "C" int ap_ipc_export(const void* dev_ptr, ap_ipc_handle_t* out) {
    if (!dev_ptr || !out) return AP_EINVAL;
    static_assert(sizeof(cudaIpcMemHandle_t) <= sizeof out->handle, "IPC handle size");
    cudaPointerAttributes attr{};
    AP_CUDA_TRY(cudaPointerGetAttributes(&attr, dev_ptr));
    if (attr.type != cudaMemoryTypeDevice) return AP_EINVAL;
    ap_device_guard g(attr.device);
    CUdeviceptr base = 0;
    size_t size = 0;
    int rc = alloc_range(dev_ptr, &base, &size);
    if (rc) return rc;
    cudaIpcMemHandle_t h;
    AP_CUDA_TRY(cudaIpcGetMemHandle(&h, (void*)base));
    ap_ipc_handle_t r{};
    memcpy(r.handle, &h, sizeof h);
    r.offset = (uint64_t)((CUdeviceptr)dev_ptr - base);
    r.bytes = (uint64_t)size - r.offset;
    r.device = attr.device;
    r.pid = (int32_t)getpid();
    *out = r;
    return AP_OK;
}

extern "C" int ap_ipc_import(const ap_ipc_handle_t* h, int device, void** dev_ptr) {
    if (!h || !dev_ptr) return AP_EINVAL;
    ap_device_guard g(device);
    cudaIpcMemHandle_t mh;
    memcpy(&mh, h->handle, sizeof mh);
    void* base = nullptr;
    AP_CUDA_TRY(cudaIpcOpenMemHandle(&base, mh, cudaIpcMemLazyEnablePeerAccess));
    *dev_ptr = (uint8_t*)base + h->offset;
    return AP_OK;
}

extern "C" int ap_ipc_close(void* dev_ptr) {
    if (!dev_ptr) return AP_EINVAL;
    CUdeviceptr base = 0;
    size_t size = 0;
    int rc = alloc_range(dev_ptr, &base, &size);
    if (rc) return rc;
    AP_CUDA_TRY(cudaIpcCloseMemHandle((void*)base));
    return AP_OK;
}

/* ------------------------------------------------------ the G partitions */
struct ap_mgpu_part {
    int device = 0;
    ap_cache_t cache = nullptr;
    ap_region_t region = 0;
    cudaStream_t stream = nullptr;
    cudaEvent_t start = nullptr, done = nullptr;
    /* per-GPU inputs: target, LSH parameters, bucket index */
    uint8_t* target = nullptr;
    int16_t* proj = nullptr;
    int32_t* bias = nullptr;
    uint32_t* offsets = nullptr;
    uint32_t* ids = nullptr;
};

struct ap_mgpu_s {
    std::vector<ap_mgpu_part> part;
    const void* file = nullptr;
    uint64_t bytes = 0;
    uint32_t* winners = nullptr; /* on the root (part[0].device) */
    uint64_t winners_blocks = 0;
    cudaEvent_t t0 = nullptr, t1 = nullptr;
    /* the inputs the per-GPU buffers hold (re-uploaded when they change) */
    ap_mgpu_collage_in prev{};
    std::vector<uint8_t> prev_target;
    std::vector<int16_t> prev_proj;
    std::vector<int32_t> prev_bias;
    bool have_prev = false;
};

static void free_inputs(ap_mgpu_part& p) {
    ap_device_guard g(p.device);
    cudaFree(p.target);
    cudaFree(p.proj);
    cudaFree(p.bias);
    cudaFree(p.offsets);
    cudaFree(p.ids);
    p.target = nullptr;
    p.proj = nullptr;
    p.bias = nullptr;
    p.offsets = nullptr;
    p.ids = nullptr;
}

extern "C" int ap_mgpu_destroy(ap_mgpu_t m) {
    if (!m) return AP_EINVAL;
    int rc = AP_OK;
    for (auto& p : m->part) {
        ap_device_guard g(p.device);
        if (p.stream) cudaStreamSynchronize(p.stream);
        free_inputs(p);
        if (p.cache) {
            int r1 = ap_munmap(p.cache, p.region);
            int r2 = ap_cache_destroy(p.cache);
            if (!rc) rc = r1 ? r1 : r2;
        }
        if (p.start) cudaEventDestroy(p.start);
        if (p.done) cudaEventDestroy(p.done);
        if (p.stream) cudaStreamDestroy(p.stream);
    }
    if (!m->part.empty()) {
        ap_device_guard g(m->part[0].device);
        cudaFree(m->winners);
        if (m->t0) cudaEventDestroy(m->t0);
        if (m->t1) cudaEventDestroy(m->t1);
    }
    delete m;
    return rc;
}

extern "C" int ap_mgpu_create(int ngpu, const int* devices, const void* host_file, uint64_t bytes,
                              uint64_t frames_per_gpu, uint32_t page_size, ap_mgpu_t* out) {
    if (ngpu < 1 || ngpu > AP_MGPU_MAX || !devices || !host_file || !bytes || !out) return AP_EINVAL;
    int ndev = 0;
    AP_CUDA_TRY(cudaGetDeviceCount(&ndev));
    for (int i = 0; i < ngpu; ++i)
        if (devices[i] < 0 || devices[i] >= ndev) return AP_EINVAL;
    ap_mgpu_s* m = new ap_mgpu_s();
    m->file = host_file;
    m->bytes = bytes;
    m->part.resize(ngpu);
    const int root = devices[0];
    int rc = AP_OK;
    for (int i = 0; i < ngpu && rc == AP_OK; ++i) {
        ap_mgpu_part& p = m->part[i];
        p.device = devices[i];
        ap_device_guard g(p.device);
        if (p.device != root) {
            /* the partition's kernels fold winners into the root's memory */
            int ok = 0;
            if (cudaDeviceCanAccessPeer(&ok, p.device, root) != cudaSuccess || !ok) {
                rc = AP_EINVAL;
                break;
            }
            cudaError_t e = cudaDeviceEnablePeerAccess(root, 0);
            if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
            else if (e != cudaSuccess) {
                cudaGetLastError();
                rc = AP_ECUDA;
                break;
            }
        }
        if (cudaStreamCreateWithFlags(&p.stream, cudaStreamNonBlocking) != cudaSuccess ||
            cudaEventCreate(&p.start) != cudaSuccess || cudaEventCreate(&p.done) != cudaSuccess) {
            cudaGetLastError();
            rc = AP_ECUDA;
            break;
        }
        rc = ap_cache_create(frames_per_gpu, page_size, p.device, &p.cache);
        if (rc == AP_OK) rc = ap_mmap(p.cache, host_file, bytes, &p.region);
        if (rc != AP_OK && p.cache) {
            ap_cache_destroy(p.cache);
            p.cache = nullptr;
        }
    }
    if (rc == AP_OK) {
        ap_device_guard g(root);
        if (cudaEventCreate(&m->t0) != cudaSuccess || cudaEventCreate(&m->t1) != cudaSuccess) {
            cudaGetLastError();
            rc = AP_ECUDA;
        }
    }
    if (rc != AP_OK) {
        ap_mgpu_destroy(m);
        return rc;
    }
    *out = m;
    return AP_OK;
}

/* Upload the target and LSH parameters and build the bucket index on every
 * GPU (each GPU indexes the file through its own cache's zero-copy alias). */
static int prepare_inputs(ap_mgpu_s* m, const ap_mgpu_collage_in* in) {
    const uint64_t tbytes = (uint64_t)in->W * in->H * 3;
    const uint64_t lk = (uint64_t)in->L * in->K;
    const bool same =
        m->have_prev && !memcmp(&m->prev, in, sizeof *in) && m->prev_target.size() == tbytes &&
        !memcmp(m->prev_target.data(), in->target_host, tbytes) &&
        m->prev_proj.size() == lk * 768 &&
        (lk == 0 || (!memcmp(m->prev_proj.data(), in->proj_host, lk * 768 * 2) &&
                     !memcmp(m->prev_bias.data(), in->bias_host, lk * 4)));
    if (same) return AP_OK;
    const uint64_t B1 = (1ull << in->bucket_bits) + 1;
    for (auto& p : m->part) {
        free_inputs(p);
        ap_device_guard g(p.device);
        if (cudaMalloc(&p.target, tbytes) != cudaSuccess ||
            cudaMalloc(&p.proj, (lk ? lk : 1) * 768 * 2) != cudaSuccess ||
            cudaMalloc(&p.bias, (lk ? lk : 1) * 4) != cudaSuccess ||
            cudaMalloc(&p.offsets, in->L * B1 * 4) != cudaSuccess ||
            cudaMalloc(&p.ids, in->L * in->N * 4) != cudaSuccess) {
            cudaGetLastError();
            free_inputs(p);
            return AP_ENOMEM;
        }
        AP_CUDA_TRY(cudaMemcpy(p.target, in->target_host, tbytes, cudaMemcpyHostToDevice));
        if (lk) {
            AP_CUDA_TRY(cudaMemcpy(p.proj, in->proj_host, lk * 768 * 2, cudaMemcpyHostToDevice));
            AP_CUDA_TRY(cudaMemcpy(p.bias, in->bias_host, lk * 4, cudaMemcpyHostToDevice));
        }
        int rc = ap_lsh_build_index(p.cache, p.region, in->N, in->rec_stride, in->L, in->K,
                                    in->bucket_bits, in->w, p.proj, p.bias, p.offsets, p.ids,
                                    p.stream);
        if (rc) return rc;
    }
    m->prev = *in;
    m->prev_target.assign(in->target_host, in->target_host + tbytes);
    m->prev_proj.assign(in->proj_host, in->proj_host + lk * 768);
    m->prev_bias.assign(in->bias_host, in->bias_host + lk);
    m->have_prev = true;
    return AP_OK;
}

extern "C" int ap_mgpu_collage(ap_mgpu_t m, const ap_mgpu_collage_in* in, uint32_t* winners_host,
                               ap_mgpu_report* rep) {
    if (!m || !in || !winners_host || !in->target_host) return AP_EINVAL;
    if (in->W == 0 || in->H == 0 || in->W % 32 || in->H % 32 || in->L == 0) return AP_EINVAL;
    if (in->K && (!in->proj_host || !in->bias_host)) return AP_EINVAL;
    if (in->bucket_bits < 1 || in->bucket_bits > 30) return AP_EINVAL;
    if (in->partition != AP_PART_BLOCKS && in->partition != AP_PART_RECORDS &&
        in->partition != AP_PART_UNITS)
        return AP_EINVAL;
    const bool units = in->schedule == AP_SCHED_TABLE || in->schedule == AP_SCHED_TABLE_MH;
    if (in->partition != AP_PART_BLOCKS && !units) return AP_EINVAL;
    const int G = (int)m->part.size();
    const uint64_t nb = (uint64_t)(in->W / 32) * (in->H / 32);
    if (in->partition == AP_PART_BLOCKS && nb < (uint64_t)G) return AP_EINVAL;
    if (in->partition == AP_PART_RECORDS && in->N < (uint64_t)G) return AP_EINVAL;
    int rc = prepare_inputs(m, in);
    if (rc) return rc;
    const int root = m->part[0].device;
    {
        ap_device_guard g(root);
        if (m->winners_blocks < nb) {
            cudaFree(m->winners);
            m->winners = nullptr;
            m->winners_blocks = 0;
            if (cudaMalloc(&m->winners, nb * 8) != cudaSuccess) {
                cudaGetLastError();
                return AP_ENOMEM;
            }
            m->winners_blocks = nb;
        }
    }
    /* cold caches, untimed */
    for (auto& p : m->part) {
        rc = ap_cache_reset(p.cache);
        if (rc) return rc;
    }
    for (auto& p : m->part) {
        ap_device_guard g(p.device);
        AP_CUDA_TRY(cudaStreamSynchronize(p.stream));
    }
    cudaStream_t rs = m->part[0].stream;
    {
        ap_device_guard g(root);
        AP_CUDA_TRY(cudaEventRecord(m->t0, rs));
        rc = ap_winners_init(m->winners, nb, rs);
        if (rc) return rc;
        AP_CUDA_TRY(cudaEventRecord(m->part[0].start, rs));
    }
    for (int i = 0; i < G; ++i) {
        ap_mgpu_part& p = m->part[i];
        ap_device_guard g(p.device);
        if (i) {
            /* the partitions start once the winners are initialised */
            AP_CUDA_TRY(cudaStreamWaitEvent(p.stream, m->part[0].start, 0));
            AP_CUDA_TRY(cudaEventRecord(p.start, p.stream));
        }
        ap_collage_in ci{};
        ci.target_dev = p.target;
        ci.W = in->W;
        ci.H = in->H;
        ci.L = in->L;
        ci.K = in->K;
        ci.bucket_bits = in->bucket_bits;
        ci.w = in->w;
        ci.proj_dev = p.proj;
        ci.bias_dev = p.bias;
        ci.offsets_dev = p.offsets;
        ci.ids_dev = p.ids;
        ci.N = in->N;
        ci.rec_stride = in->rec_stride;
        ci.group = in->group;
        ci.mode = AP_MODE_APOINTER;
        ci.schedule = in->schedule;
        ci.id_chunks = in->id_chunks;
        ci.flags = AP_COLLAGE_ACCUMULATE | AP_COLLAGE_SYSTEM;
        uint32_t* out = m->winners;
        if (in->partition == AP_PART_BLOCKS) {
            const uint64_t b0 = nb * i / G, b1 = nb * (i + 1) / G;
            ci.block_begin = b0;
            ci.block_count = b1 - b0;
            out = m->winners + 2 * b0;
        } else {
            ci.block_begin = 0;
            ci.block_count = nb;
            if (in->partition == AP_PART_RECORDS) {
                ci.id_begin = (uint32_t)(in->N * i / G);
                ci.id_end = (uint32_t)(in->N * (i + 1) / G);
                if (in->id_chunks > ci.id_end - ci.id_begin) ci.id_chunks = ci.id_end - ci.id_begin;
            } else {
                const uint64_t nu = nb * in->L;
                ci.unit_begin = nu * i / G;
                ci.unit_count = nu * (i + 1) / G - ci.unit_begin;
                if (ci.unit_count == 0) {
                    AP_CUDA_TRY(cudaEventRecord(p.done, p.stream));
                    continue;
                }
            }
        }
        rc = ap_collage_run(p.cache, p.region, &ci, out, p.stream);
        if (rc) return rc;
        AP_CUDA_TRY(cudaEventRecord(p.done, p.stream));
    }
    {
        ap_device_guard g(root);
        for (int i = 1; i < G; ++i) AP_CUDA_TRY(cudaStreamWaitEvent(rs, m->part[i].done, 0));
        AP_CUDA_TRY(cudaEventRecord(m->t1, rs));
        AP_CUDA_TRY(cudaMemcpyAsync(winners_host, m->winners, nb * 8, cudaMemcpyDeviceToHost, rs));
        AP_CUDA_TRY(cudaStreamSynchronize(rs));
    }
    if (rep) {
        ap_mgpu_report r{};
        r.nparts = G;
        float ms = 0.f;
        {
            ap_device_guard g(root);
            cudaEventElapsedTime(&ms, m->t0, m->t1);
        }
        r.seconds = ms * 1e-3;
        for (int i = 0; i < G; ++i) {
            ap_mgpu_part& p = m->part[i];
            ap_device_guard g(p.device);
            AP_CUDA_TRY(cudaStreamSynchronize(p.stream));
            float pm = 0.f;
            cudaEventElapsedTime(&pm, p.start, p.done);
            r.part_seconds[i] = pm * 1e-3;
            ap_stats_t st{};
            if (ap_cache_stats(p.cache, &st) == AP_OK) {
                r.fill_bytes[i] = st.fill_bytes;
                r.major[i] = st.major;
            }
            const int err = ap_last_device_error(p.cache);
            if (err && r.device_error == AP_OK) r.device_error = err;
        }
        *rep = r;
    }
    return AP_OK;
}

extern "C" int ap_collage_mgpu(int ngpu, const int* devices, const void* host_file, uint64_t bytes,
                               uint64_t frames_per_gpu, uint32_t page_size,
                               const ap_mgpu_collage_in* in, uint32_t* winners_host,
                               ap_mgpu_report* rep) {
    ap_mgpu_t m = nullptr;
    int rc = ap_mgpu_create(ngpu, devices, host_file, bytes, frames_per_gpu, page_size, &m);
    if (rc) return rc;
    rc = ap_mgpu_collage(m, in, winners_host, rep);
    const int rd = ap_mgpu_destroy(m);
    return rc ? rc : rd;
}
