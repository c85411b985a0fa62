// tools/gatherprobe.cu -- measurement helper (not the method): how fast can an SM gather whole B rows
// (RB = 4K bytes each, K = 64 -> 256 B, K = 128 -> 512 B) from L2 / HBM?
//   mode 0: register loads -- a group of 8 lanes reads one row with one 256-bit load per lane per 256 B,
//           U rows in flight per group (what k_spmm does);
//   mode 1: cp.async.bulk (TMA 1-D bulk copy, UBLKCP) of each row into a per-group shared-memory ring of S
//           slots, one mbarrier per slot, copies issued one batch (8 rows) ahead by the group's lanes.
// Reports GB/s of gathered row bytes.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gp gatherprobe.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

struct f8 { float4 lo, hi; };
__device__ __forceinline__ f8 ld8(const void *p) {
    f8 r;
    asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(r.lo.x), "=f"(r.lo.y), "=f"(r.lo.z), "=f"(r.lo.w), "=f"(r.hi.x), "=f"(r.hi.y), "=f"(r.hi.z),
                   "=f"(r.hi.w)
                 : "l"(p));
    return r;
}

template <int RB, int U>
__global__ void __launch_bounds__(256) k_reg(const char *__restrict__ B, const int *__restrict__ idx, int64_t per_group,
                                             float *out) {
    const int lane = threadIdx.x & 31, g = lane >> 3, gl = lane & 7;
    const int64_t grp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 8;
    const int *my = idx + grp * per_group;
    float acc = 0.f;
    constexpr int NV = RB / 256;   // 256-bit loads per lane per row
    for (int64_t q = 0; q < per_group; q += U) {
        f8 x[U][NV];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int r = __ldg(my + q + u);
#pragma unroll
            for (int v = 0; v < NV; ++v) x[u][v] = ld8(B + (size_t)r * RB + v * 256 + gl * 32);
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int v = 0; v < NV; ++v) acc += x[u][v].lo.x + x[u][v].hi.w;
    }
    (void)g;
    out[(int64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int RB, int S, int WARPS>
__global__ void __launch_bounds__(WARPS * 32, 1) k_bulk(const char *__restrict__ B, const int *__restrict__ idx,
                                                        int64_t per_group, float *out) {
    extern __shared__ __align__(128) char sm[];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, g = lane >> 3, gl = lane & 7;
    const int gw = w * 4 + g;                           // group within CTA
    char *ring = sm + (size_t)gw * S * RB;
    uint64_t *bars = reinterpret_cast<uint64_t *>(sm + (size_t)WARPS * 4 * S * RB) + gw * S;
    for (int s = gl; s < S; s += 8)
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bars + s)));
    asm volatile("fence.mbarrier_init.release.cluster;");
    __syncthreads();
    const int64_t grp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 8;
    const int *my = idx + grp * per_group;
    float acc = 0.f;
    auto issue = [&](int64_t q) {
        if (q < per_group) {
            const int r = __ldg(my + q);
            const int s = (int)(q % S);
            const uint32_t bar = smem_u32(bars + s);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(RB) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(smem_u32(ring + (size_t)s * RB)), "l"(B + (size_t)r * RB), "r"(RB), "r"(bar) : "memory");
        }
    };
    // prologue: S rows in flight
    for (int64_t q = gl; q < S; q += 8) issue(q);
    for (int64_t q0 = 0; q0 < per_group; q0 += 8) {
        for (int k = 0; k < 8; ++k) {
            const int64_t q = q0 + k;
            const int s = (int)(q % S);
            const uint32_t par = (uint32_t)((q / S) & 1);
            const uint32_t bar = smem_u32(bars + s);
            uint32_t done = 0;
            while (!done) {
                asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                             : "=r"(done) : "r"(bar), "r"(par) : "memory");
            }
            const float4 *row = reinterpret_cast<const float4 *>(ring + (size_t)s * RB);
#pragma unroll
            for (int v = 0; v < RB / 256; ++v) {
                const float4 a = row[v * 16 + gl * 2], b = row[v * 16 + gl * 2 + 1];
                acc += a.x + b.w;
            }
        }
        __syncwarp();
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue(q0 + S + gl);    // refill the batch just consumed (S is a multiple of 8)
        if (S > 8) {}
    }
    out[(int64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main(int argc, char **argv) {
    const int64_t ws_mb = argc > 1 ? atoll(argv[1]) : 64;       // gather window (MB)
    const int mode = argc > 2 ? atoi(argv[2]) : 0;
    const int rb = argc > 3 ? atoi(argv[3]) : 256;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t B_bytes = 1ll << 30;
    char *B;
    cudaMalloc(&B, B_bytes);
    cudaMemset(B, 0, B_bytes);
    const int64_t rows = ws_mb * (1 << 20) / rb;
    const int WARPS = 12;
    const int bps = argc > 4 ? atoi(argv[4]) : 8;
    const int blocks_reg = sms * bps, threads = 256;
    const int64_t groups_reg = (int64_t)blocks_reg * threads / 8;
    const int64_t groups_bulk = (int64_t)sms * WARPS * 4;
    const int64_t per_group = 4096;
    const int64_t ng = groups_reg > groups_bulk ? groups_reg : groups_bulk;
    int *h = (int *)malloc(ng * per_group * sizeof(int));
    uint64_t x = 88172645463325252ull;
    for (int64_t i = 0; i < ng * per_group; ++i) {
        x ^= x << 13; x ^= x >> 7; x ^= x << 17;
        h[i] = (int)(x % rows);
    }
    int *idx;
    cudaMalloc(&idx, ng * per_group * sizeof(int));
    cudaMemcpy(idx, h, ng * per_group * sizeof(int), cudaMemcpyHostToDevice);
    float *out;
    cudaMalloc(&out, (size_t)ng * 8 * sizeof(float) * 2);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int m = (mode < 0 ? 0 : mode); m <= (mode < 0 ? 3 : mode); ++m) {
        float best = 1e30f;
        int64_t bytes = 0;
        for (int rep = 0; rep < 5; ++rep) {
            cudaEventRecord(e0);
            if (m == 0 || m == 2) {
                if (rb == 256) {
                    if (m == 0) k_reg<256, 4><<<blocks_reg, threads>>>(B, idx, per_group, out);
                    else k_reg<256, 8><<<blocks_reg, threads>>>(B, idx, per_group, out);
                } else {
                    if (m == 0) k_reg<512, 2><<<blocks_reg, threads>>>(B, idx, per_group, out);
                    else k_reg<512, 4><<<blocks_reg, threads>>>(B, idx, per_group, out);
                }
                bytes = groups_reg * per_group * rb;
            } else {
                if (rb == 256) {
                    if (m == 1) {
                        auto k = k_bulk<256, 16, WARPS>;
                        const int smem = WARPS * 4 * 16 * 256 + WARPS * 4 * 16 * 8;
                        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                        k<<<sms, WARPS * 32, smem>>>(B, idx, per_group, out);
                    } else {
                        auto k = k_bulk<256, 8, WARPS>;
                        const int smem = WARPS * 4 * 8 * 256 + WARPS * 4 * 8 * 8;
                        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                        k<<<sms, WARPS * 32, smem>>>(B, idx, per_group, out);
                    }
                } else {
                    auto k = k_bulk<512, 8, WARPS>;
                    const int smem = WARPS * 4 * 8 * 512 + WARPS * 4 * 8 * 8;
                    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                    k<<<sms, WARPS * 32, smem>>>(B, idx, per_group, out);
                }
                bytes = groups_bulk * per_group * rb;
            }
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        cudaError_t err = cudaGetLastError();
        printf("bps=%d ws=%lld MB rb=%d mode=%d (%s): %.3f ms, %.1f GB/s, %.2f rows/clk/SM@1.9GHz %s\n", bps, (long long)ws_mb, rb, m,
               m == 0 ? "reg U=4/2" : m == 2 ? "reg U=8/4" : m == 1 ? "bulk S=16" : "bulk S=8", best,
               bytes / (best * 1e-3) / 1e9, bytes / rb / (best * 1e-3) / 1.9e9 / sms, cudaGetErrorString(err));
    }
    return 0;
}
