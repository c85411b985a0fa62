// tools/dsmemprobe.cu -- measurement helper (not the method): how fast can the SMs of a thread-block cluster
// gather whole B rows (RB bytes) out of each other's shared memory (distributed shared memory, DSMEM), and does
// that traffic add to L2->SM gathers?  A cluster of CS CTAs (1 per SM) fills its shared memory with NROWS rows
// each; then every 8-lane group reads random rows of random CTAs of its cluster (ld.shared::cluster.v4, via
// mapa), MIX of every 8 reads going to an L2-resident global buffer instead.  Reports GB/s of gathered bytes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o dsmemprobe dsmemprobe.cu
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

namespace cg = cooperative_groups;

__device__ __forceinline__ float4 ld_dsmem(uint32_t cluster_addr) {
    float4 r;
    asm volatile("ld.shared::cluster.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "r"(cluster_addr));
    return r;
}
__device__ __forceinline__ uint32_t map_rank(uint32_t smem_addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_addr), "r"(rank));
    return r;
}

template <int RB, int U>
__global__ void k_dsmem(const float4 *__restrict__ gbuf, int64_t grows, int nrows, int iters, int mix, float *out) {
    extern __shared__ __align__(16) float4 sm[];
    cg::cluster_group cluster = cg::this_cluster();
    const int cs = (int)cluster.num_blocks();
    for (int i = threadIdx.x; i < nrows * RB / 16; i += blockDim.x) sm[i] = make_float4(1.f, 2.f, 3.f, (float)i);
    cluster.sync();
    const int lane = threadIdx.x & 31, gl = lane & 7;
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
    uint32_t x = 0x9E3779B9u * (blockIdx.x * blockDim.x + threadIdx.x + 1) | 1u;
    // one random stream per 8-lane group (lanes of a group share the row)
    uint32_t gx = __shfl_sync(0xffffffffu, x, lane & ~7);
    float acc = 0.f;
    for (int it = 0; it < iters; ++it) {
        float4 v[U][RB / 128];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            gx ^= gx << 13; gx ^= gx >> 17; gx ^= gx << 5;
            const bool global = (int)(gx & 7u) < mix;
            if (global) {
                const int64_t row = (int64_t)((gx >> 3) % (uint32_t)grows);
#pragma unroll
                for (int k = 0; k < RB / 128; ++k) v[u][k] = __ldg(gbuf + row * (RB / 16) + k * 8 + gl);
            } else {
                const uint32_t rank = (gx >> 3) % (uint32_t)cs;
                const uint32_t row = (gx >> 8) % (uint32_t)nrows;
                const uint32_t a = map_rank(base + row * RB, rank);
#pragma unroll
                for (int k = 0; k < RB / 128; ++k) v[u][k] = ld_dsmem(a + (k * 8 + gl) * 16);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int k = 0; k < RB / 128; ++k) acc += v[u][k].x + v[u][k].w;
    }
    cluster.sync();
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main(int argc, char **argv) {
    const int cs = argc > 1 ? atoi(argv[1]) : 8;          // cluster size
    const int mix = argc > 2 ? atoi(argv[2]) : 0;         // of 8 reads, how many go to the global buffer
    const int threads = argc > 3 ? atoi(argv[3]) : 512;
    constexpr int RB = 512;
    const int nrows = 400;                                 // 400 x 512 B = 200 KB per CTA
    const size_t smem = (size_t)nrows * RB;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t grows = (64ll << 20) / RB;               // 64 MB L2-resident global buffer
    float4 *g;
    cudaMalloc(&g, grows * RB);
    cudaMemset(g, 0, grows * RB);
    float *out;
    cudaMalloc(&out, (size_t)sms * 2 * threads * sizeof(float));
    auto kern = k_dsmem<RB, 4>;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (cs > 8) cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = cs;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int nclusters = 0;
    cfg.gridDim = dim3(cs);
    cudaOccupancyMaxActiveClusters(&nclusters, kern, &cfg);
    if (nclusters <= 0) { printf("cs=%d: no cluster fits (%s)\n", cs, cudaGetErrorString(cudaGetLastError())); return 1; }
    cfg.gridDim = dim3(nclusters * cs);
    const int iters = 2000;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 4; ++rep) {
        cudaEventRecord(e0);
        cudaLaunchKernelEx(&cfg, kern, (const float4 *)g, grows, nrows, iters, mix, out);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    const double rows = (double)nclusters * cs * (threads / 8) * iters * 4;
    printf("cluster=%d clusters=%d ctas=%d threads=%d mix=%d/8 global: %.3f ms, %.1f GB/s gathered (%s)\n", cs,
           nclusters, nclusters * cs, threads, mix, best, rows * RB / (best * 1e-3) / 1e9,
           cudaGetErrorString(cudaGetLastError()));
    return 0;
}
