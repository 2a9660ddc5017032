// atomic_ceiling.cu — the ceiling of the minor-fault regime (M2r, SURVEY.md
// §8(d)): every apointer read there is one warp-aggregated link (an acquire
// add on a PTE) and one unlink (a release add) on 8-B entries of a 16 384-entry
// page table, plus one 4-B gather from the resident GiB.  This measures the
// same memory traffic with no page-cache logic around it, all SMs, every
// thread its own random PTE per step (the M2r pattern: each read leaves its
// page, warps are not aggregated because the 32 lanes hit 32 random pages):
//   (a) relaxed add + relaxed add per step          (the atomics alone, no ordering)
//   (b) acquire add + release add per step          (the link/unlink pair's ordering)
//   (c) (b) + the 4-B gather the read itself does   (the whole M2r access)
//   (d) the 4-B gather alone                        (the raw twin)
// Reports G steps/s (= G reads/s of M2r).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o atomic_ceiling atomic_ceiling.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
    uint64_t z = x + 0x9e3779b97f4a7c15ull;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}

template <int MODE>
__global__ void __launch_bounds__(512) k_atom(unsigned long long* pte, uint32_t npte,
                                              const uint32_t* data, uint64_t nwords, uint32_t reads,
                                              uint64_t* out) {
    const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint64_t h = 0;
    for (uint32_t i = 0; i < reads; ++i) {
        const uint64_t r = sm64((t << 24) ^ i);
        const uint64_t p = r % npte;
        if (MODE == 0) {
            unsigned long long o;
            asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], 1;" : "=l"(o) : "l"(pte + p) : "memory");
            h += o;
            asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(pte + p), "l"(~0ull) : "memory");
        } else if (MODE == 1 || MODE == 2) {
            unsigned long long o;
            asm volatile("atom.acquire.gpu.global.add.u64 %0, [%1], 1;" : "=l"(o) : "l"(pte + p) : "memory");
            h += o;
            if (MODE == 2) h += __ldcg(data + (((r >> 20) ^ o) % nwords));
            asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(pte + p), "l"(~0ull) : "memory");
        } else {
            h += __ldcg(data + ((r >> 20) % nwords));
        }
    }
    out[t] = h;
}

int main() {
    const uint32_t npte = 16384;
    const uint64_t nwords = (1ull << 30) / 4;
    const int grid = 4 * 148, block = 512;
    const uint32_t reads = 8;
    unsigned long long* pte;
    uint32_t* data;
    uint64_t* out;
    CK(cudaMalloc(&pte, npte * 8));
    CK(cudaMemset(pte, 0, npte * 8));
    CK(cudaMalloc(&data, nwords * 4));
    CK(cudaMemset(data, 1, nwords * 4));
    CK(cudaMalloc(&out, (size_t)grid * block * 8));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const char* names[4] = {"relaxed add + relaxed add", "acquire add + release add",
                            "acquire add + 4-B gather + release add", "4-B gather alone"};
    for (int mode = 0; mode < 4; ++mode) {
        float best = 1e30f;
        for (int rep = 0; rep < 6; ++rep) {
            cudaEventRecord(a);
            switch (mode) {
                case 0: k_atom<0><<<grid, block>>>(pte, npte, data, nwords, reads, out); break;
                case 1: k_atom<1><<<grid, block>>>(pte, npte, data, nwords, reads, out); break;
                case 2: k_atom<2><<<grid, block>>>(pte, npte, data, nwords, reads, out); break;
                default: k_atom<3><<<grid, block>>>(pte, npte, data, nwords, reads, out);
            }
            cudaEventRecord(b);
            CK(cudaEventSynchronize(b));
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (rep && ms < best) best = ms;
        }
        const double steps = (double)grid * block * reads;
        printf("%-40s %8.2f G steps/s  (%.3f ms for %.0f steps)\n", names[mode],
               steps / (best * 1e-3) / 1e9, best, steps);
    }
    return 0;
}
