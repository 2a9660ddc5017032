// fill_microbench.cu — host-link fill A/B for the fault path (S8):
//   (a) warp zero-copy 16-B loads + stores (what fill_page does),
//   (b) TMA bulk copies host->smem->HBM per warp (cp.async.bulk + mbarrier).
// Copies `bytes` from pinned, mapped host memory into device memory in
// `chunk`-byte pieces handed to warps round-robin, and prints GB/s.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fill_mb fill_microbench.cu
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__global__ void __launch_bounds__(512) k_ldg(const uint4* __restrict__ src, uint4* __restrict__ dst,
                                             uint64_t nchunks, uint32_t chunk) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const unsigned lane = threadIdx.x & 31;
    const uint32_t nvec = chunk / 16;
    for (uint64_t c = warp; c < nchunks; c += nw) {
        const uint4* s = src + c * nvec;
        uint4* d = dst + c * nvec;
        for (uint32_t i = lane; i < nvec; i += 32 * 8) {
            uint4 v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) if (i + 32 * u < nvec) v[u] = __ldcs(s + i + 32 * u);
#pragma unroll
            for (int u = 0; u < 8; ++u) if (i + 32 * u < nvec) __stcg(d + i + 32 * u, v[u]);
        }
    }
}

template <int FLAV, int U>
__global__ void __launch_bounds__(512) k_ldg2(const uint4* __restrict__ src, uint4* __restrict__ dst,
                                              uint64_t nchunks, uint32_t chunk) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const unsigned lane = threadIdx.x & 31;
    const uint32_t nvec = chunk / 16;
    for (uint64_t c = warp; c < nchunks; c += nw) {
        const uint4* s = src + c * nvec;
        uint4* d = dst + c * nvec;
        for (uint32_t i = lane; i < nvec; i += 32 * U) {
            uint4 v[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint4* p = s + i + 32 * u;
                if (FLAV == 0) v[u] = __ldcs(p);
                else if (FLAV == 1) asm volatile("ld.global.nc.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(p));
                else if (FLAV == 2) asm volatile("ld.global.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(p));
                else asm volatile("ld.global.cg.L2::128B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(p));
            }
#pragma unroll
            for (int u = 0; u < U; ++u) __stcg(d + i + 32 * u, v[u]);
        }
    }
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

// per warp: NBUF buffers of `chunk` bytes + NBUF mbarriers
template <int NBUF>
__global__ void __launch_bounds__(512) k_tma(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                             uint64_t nchunks, uint32_t chunk) {
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ __align__(8) uint64_t mbar[16][NBUF];
    const unsigned wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    uint8_t* buf = smem + (size_t)wid * NBUF * chunk;
    if (lane == 0) {
        for (int b = 0; b < NBUF; ++b)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[wid][b])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t phase[NBUF] = {};
    uint64_t c = warp;
    int b = 0;
    // prologue: issue NBUF loads
    uint64_t inflight[NBUF];
    for (int k = 0; k < NBUF; ++k) inflight[k] = ~0ull;
    for (int k = 0; k < NBUF && c < nchunks; ++k, c += nw) {
        if (lane == 0) {
            uint32_t mb = smem_u32(&mbar[wid][k]);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(chunk) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(smem_u32(buf + k * chunk)), "l"(src + c * chunk), "r"(chunk), "r"(mb) : "memory");
        }
        inflight[k] = c;
    }
    while (true) {
        if (inflight[b] == ~0ull) break;
        // wait for buffer b
        if (lane == 0) {
            uint32_t mb = smem_u32(&mbar[wid][b]);
            uint32_t done = 0;
            while (!done) {
                asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                             : "=r"(done) : "r"(mb), "r"(phase[b]) : "memory");
            }
            // store smem -> global
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                         ::"l"(dst + inflight[b] * chunk), "r"(smem_u32(buf + b * chunk)), "r"(chunk) : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        }
        phase[b] ^= 1;
        inflight[b] = ~0ull;
        if (c < nchunks) {
            if (lane == 0) {
                uint32_t mb = smem_u32(&mbar[wid][b]);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(chunk) : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(smem_u32(buf + b * chunk)), "l"(src + c * chunk), "r"(chunk), "r"(mb) : "memory");
            }
            inflight[b] = c;
            c += nw;
        }
        b = (b + 1) % NBUF;
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    __syncwarp();
}

int main(int argc, char** argv) {
    const uint64_t bytes = 1ull << 30;
    uint8_t* h = nullptr;
    CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(h, 1, bytes);
    uint8_t* hd = nullptr;
    CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
    uint8_t* d = nullptr;
    CK(cudaMalloc(&d, bytes));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float ms = 0;
    for (int i = 0; i < 3; ++i) {
        cudaEventRecord(e0);
        CK(cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice));
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
    }
    printf("memcpy H2D            %.2f GB/s\n", bytes / ms / 1e6);
    for (uint32_t chunk : {4096u, 16384u, 65536u}) {
        for (int blocks : {148, 296}) {
            uint64_t n = bytes / chunk;
            for (int i = 0; i < 3; ++i) {
                cudaEventRecord(e0);
                k_ldg<<<blocks, 512>>>((const uint4*)hd, (uint4*)d, n, chunk);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                cudaEventElapsedTime(&ms, e0, e1);
            }
            CK(cudaGetLastError());
            printf("ldg   chunk %6u grid %3d  %.2f GB/s\n", chunk, blocks, bytes / ms / 1e6);
        }
    }
    {
        const uint32_t chunk = 4096;
        const uint64_t n = bytes / chunk;
        auto run = [&](auto kern, const char* name) {
            for (int i = 0; i < 3; ++i) {
                cudaEventRecord(e0);
                kern<<<148, 512>>>((const uint4*)hd, (uint4*)d, n, chunk);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                cudaEventElapsedTime(&ms, e0, e1);
            }
            printf("%-28s %.2f GB/s\n", name, bytes / ms / 1e6);
        };
        run(k_ldg2<0, 8>, "ld.cs unroll8");
        run(k_ldg2<0, 4>, "ld.cs unroll4");
        run(k_ldg2<1, 8>, "ld.nc.L2::256B unroll8");
        run(k_ldg2<2, 8>, "ld.L2::256B unroll8");
        run(k_ldg2<3, 8>, "ld.cg.L2::128B unroll8");
    }
    for (uint32_t chunk : {2048u, 4096u, 8192u}) {
        size_t sm = 16 * 2 * chunk;
        if (sm > 200 * 1024) continue;
        CK(cudaFuncSetAttribute(k_tma<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
        uint64_t n = bytes / chunk;
        for (int i = 0; i < 3; ++i) {
            cudaEventRecord(e0);
            k_tma<2><<<148, 512, sm>>>(hd, d, n, chunk);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&ms, e0, e1);
        }
        CK(cudaGetLastError());
        printf("tma2  chunk %6u grid 148  %.2f GB/s\n", chunk, bytes / ms / 1e6);
    }
    // correctness spot check
    uint8_t probe[16];
    CK(cudaMemcpy(probe, d + bytes - 16, 16, cudaMemcpyDeviceToHost));
    printf("probe %d\n", probe[0]);
    return 0;
}
