// ubench_chain.cu — single-thread dependent-chain latency probes for the DFS critical chain
// (sm_100a).  Every figure is (kernel time) / (iterations) of a chain in which iteration k+1's
// address depends on iteration k's result, timed with CUDA events (no in-kernel clock reads,
// which ptxas may hoist above the consuming instruction).
//
//   ld_hbm       ld.global.nc chain over a 4 GB table (HBM misses)
//   ld_l2        ld.global.cg chain over a 4 MB table (L2 hits)
//   atom         atom.global.or chain over the 4 MB table (L2 atomics, result consumed)
//   atom+ld_l2   chain through the atomic; an independent L2 load issued right after it each
//                iteration and consumed one iteration later (does the load wait for the atomic?)
//   ld_l2+atom   chain through the L2 load; an independent atomic issued right BEFORE it
//   atom+hbm     chain through the atomic; independent HBM load issued after it
//   atom+hbm+rel chain through the atomic; independent HBM load, then atom.release.cta.shared
//                (does MEMBAR.ALL.CTA wait for the outstanding HBM load?)
//   atom+rel     chain through the atomic, then atom.release.cta.shared each iteration
//   ld_l2+rel    chain through L2 loads; a release smem atomic after each load is issued
//   ld_l2+ld_l2  two independent L2 loads per iteration (MLP sanity check)
//   atom_then_hbm(+rel)  as atom+hbm(+rel) with the HBM load ordered AFTER the atomic in SASS
//   hbmchain_then_atom   chain through HBM loads; an independent atomic issued after each load
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench_chain ubench_chain.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t ldnc(const uint32_t* p) {
    uint32_t v; asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(v) : "l"(p)); return v;
}
__device__ __forceinline__ uint32_t ldnc_m(const uint32_t* p) {   // ordered after prior asm
    uint32_t v; asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ uint32_t ldcg(const uint32_t* p) {
    uint32_t v; asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p)); return v;
}
__device__ __forceinline__ uint32_t atom_or(uint32_t* p, uint32_t b) {
    uint32_t v; asm volatile("atom.global.or.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "r"(b) : "memory"); return v;
}
__device__ __forceinline__ void smem_rel_add(uint32_t a, uint32_t v) {
    asm volatile("atom.release.cta.shared.add.u32 _, [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

constexpr size_t kBig = (size_t)1 << 30;     // words (4 GB)
constexpr uint32_t kSmall = 1u << 20;        // words (4 MB)

__global__ void chain(int mode, const uint32_t* big, uint32_t* small, int iters, uint32_t* out) {
    __shared__ uint32_t sw;
    sw = 0;
    const uint32_t sa = (uint32_t)__cvta_generic_to_shared(&sw);
    uint32_t x = 1, y = 7, acc = 0, pend = 0;
    for (int k = 0; k < iters; ++k) {
        switch (mode) {
            case 0: x = ldnc(big + ((size_t)x * 32u) % kBig); break;
            case 1: x = ldcg(small + x % kSmall); break;
            case 2: x = atom_or(small + x % kSmall, 0u); break;
            case 3: { uint32_t o = atom_or(small + x % kSmall, 0u); uint32_t l = ldcg(small + (y + 4099u * k) % kSmall);
                      acc += pend; pend = l; x = o; } break;
            case 4: { uint32_t o = atom_or(small + (y + 8191u * k) % kSmall, 0u); uint32_t l = ldcg(small + x % kSmall);
                      acc += pend; pend = o; x = l; } break;
            case 5: { uint32_t o = atom_or(small + x % kSmall, 0u); uint32_t l = ldnc(big + ((size_t)(y + 4099u * k) * 32u) % kBig);
                      acc += pend; pend = l; x = o; } break;
            case 6: { uint32_t o = atom_or(small + x % kSmall, 0u); uint32_t l = ldnc(big + ((size_t)(y + 4099u * k) * 32u) % kBig);
                      smem_rel_add(sa, 1u); acc += pend; pend = l; x = o; } break;
            case 7: { x = atom_or(small + x % kSmall, 0u); smem_rel_add(sa, 1u); } break;
            case 8: { x = ldcg(small + x % kSmall); smem_rel_add(sa, 1u); } break;
            case 10: { uint32_t o = atom_or(small + x % kSmall, 0u); uint32_t l = ldnc_m(big + ((size_t)(y + 4099u * k) * 32u) % kBig);
                      acc += pend; pend = l; x = o; } break;
            case 11: { uint32_t o = atom_or(small + x % kSmall, 0u); uint32_t l = ldnc_m(big + ((size_t)(y + 4099u * k) * 32u) % kBig);
                      smem_rel_add(sa, 1u); acc += pend; pend = l; x = o; } break;
            case 12: { uint32_t l = ldnc_m(big + ((size_t)x * 32u) % kBig); uint32_t o = atom_or(small + (y + 8191u * k) % kSmall, 0u);
                      acc += pend; pend = o; x = l; } break;
            case 9: { uint32_t a = ldcg(small + x % kSmall); uint32_t b = ldcg(small + (x + 77777u) % kSmall); x = a ^ (b & 0u) ; acc += b; } break;
        }
    }
    out[0] = x + acc + pend + sw;
}

__global__ void fill(uint32_t* p, size_t n, uint32_t salt) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        uint64_t h = (i + salt) * 0x9E3779B97F4A7C15ull;
        h ^= h >> 29; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 32;
        p[i] = (uint32_t)h;
    }
}

int main() {
    uint32_t *big, *small, *out;
    cudaMalloc(&big, kBig * 4); cudaMalloc(&small, (size_t)kSmall * 4); cudaMalloc(&out, 64);
    fill<<<1184, 256>>>(big, kBig, 1); fill<<<148, 256>>>(small, kSmall, 2);
    cudaDeviceSynchronize();
    const char* names[] = {"ld_hbm", "ld_l2", "atom", "atom+ld_l2", "ld_l2+atom", "atom+hbm", "atom+hbm+rel",
                           "atom+rel", "ld_l2+rel", "ld_l2+ld_l2", "atom_then_hbm", "atom_then_hbm+rel",
                           "hbmchain_then_atom"};
    int clk = 0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    printf("{");
    for (int mode = 0; mode < 13; ++mode) {
        const int iters = 20000;
        chain<<<1, 1>>>(mode, big, small, 1000, out);
        cudaEventRecord(e0);
        chain<<<1, 1>>>(mode, big, small, iters, out);
        cudaEventRecord(e1);
        cudaError_t e = cudaEventSynchronize(e1);
        if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
        float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
        const double ns = ms * 1e6 / iters;
        printf("%s\"%s\": {\"ns\": %.1f, \"cyc_at_max_clock\": %.0f}", mode ? ", " : "", names[mode], ns, ns * clk / 1e6);
    }
    printf(", \"clock_khz\": %d}\n", clk);
    return 0;
}
