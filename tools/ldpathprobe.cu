// tools/ldpathprobe.cu -- measurement helper (not the method): the SM's load-path ceiling for B-row gathers.
//
// k_spmm moves 4K bytes of B per nnz into registers (every nnz reads its whole B row).  How many bytes per SM
// clock can an SM take in this way, and does it depend on where the rows live (L1-resident, L2-resident, HBM)
// or on the shape of the load instructions?  Each thread block gathers random rows of RB bytes from a window of
// `window` bytes and sums one word per vector (so the loads cannot be elided).  Shapes (one warp instruction):
//   0  k_spmm's shape: 8-lane groups, one 256-bit load per lane (LDG.E.ENL2.256): 4 rows x 256 B = 8 lines
//   1  warp per row, 128-bit loads: 512 B contiguous = 4 lines
//   2  warp per line, 32-bit loads: 128 B = 1 line
//   3  4-lane groups, 256-bit loads: 8 rows x 128 B = 8 lines
//   4  shape 0 with L1::no_allocate
//   5  shared memory: rows staged once per CTA, then gathered with 128-bit LDS, warp per 512-B row (crossbar)
// Reported: GB/s and bytes per SM clock (clock64 deltas per block; the SM clock under load is what the probe
// itself sees, so power capping does not distort B/clk).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ldp ldpathprobe.cu ; run: ./ldp
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <algorithm>

struct f8 { float4 lo, hi; };
template <bool NA>
__device__ __forceinline__ f8 ld8(const void *p) {
    f8 r;
    if (NA)
        asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=f"(r.lo.x), "=f"(r.lo.y), "=f"(r.lo.z), "=f"(r.lo.w), "=f"(r.hi.x), "=f"(r.hi.y),
                       "=f"(r.hi.z), "=f"(r.hi.w) : "l"(p));
    else
        asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=f"(r.lo.x), "=f"(r.lo.y), "=f"(r.lo.z), "=f"(r.lo.w), "=f"(r.hi.x), "=f"(r.hi.y),
                       "=f"(r.hi.z), "=f"(r.hi.w) : "l"(p));
    return r;
}

// random row index stream: a multiplicative hash of a counter, nrows a power of two (2 integer ops: the probe
// must stay bound by its loads, not by index arithmetic)
__device__ __forceinline__ uint32_t hrow(uint64_t x, uint32_t nrows) {
    return ((uint32_t)x * 0x9E3779B1u) >> 7 & (nrows - 1);
}

constexpr int U = 4;   // independent row loads in flight per lane

template <int SHAPE>
__global__ void __launch_bounds__(256, 3) k_probe(const char *__restrict__ B, uint32_t nrows, int RB, int iters,
                                                  float *out, unsigned long long *cyc) {
    const int lane = threadIdx.x & 31;
    const uint64_t wid = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    float acc = 0.f;
    const long long t0 = clock64();
    if (SHAPE == 0 || SHAPE == 3 || SHAPE == 4) {
        const int G = SHAPE == 3 ? 4 : 8;              // lanes per row group, 32 B each
        const int g = lane / G, gl = lane % G;
        const int span = G * 32;                        // bytes per group instruction
        for (int it = 0; it < iters; ++it) {
            f8 x[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t r = hrow(((wid * iters + it) * U + u) * 8 + g, nrows);
                const char *p = B + (size_t)r * RB + (size_t)((it * U + u) & (RB / span - 1)) * span + gl * 32;
                x[u] = ld8<SHAPE == 4>(p);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) acc += x[u].lo.x + x[u].hi.w;
        }
    } else if (SHAPE == 1) {                            // warp per row: 512 B (4 lines) per instruction
        for (int it = 0; it < iters; ++it) {
            float4 x[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t r = hrow((wid * iters + it) * U + u, nrows);
                x[u] = __ldg(reinterpret_cast<const float4 *>(B + (size_t)r * RB) + ((it * U + u) & (RB / 512 - 1)) * 32 + lane);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) acc += x[u].x + x[u].w;
        }
    } else if (SHAPE == 2) {                            // warp per line: 128 B per instruction
        for (int it = 0; it < iters; ++it) {
            float x[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t r = hrow((wid * iters + it) * U + u, nrows);
                x[u] = __ldg(reinterpret_cast<const float *>(B + (size_t)r * RB) + ((it * U + u) & (RB / 128 - 1)) * 32 + lane);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) acc += x[u];
        }
    }
    const long long t1 = clock64();
    out[(uint64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
    if (threadIdx.x == 0) atomicMax(cyc + blockIdx.x % 1024, (unsigned long long)(t1 - t0));
}

// shape 0 with UU row loads in flight per lane and MINB CTAs per SM (in-flight bytes per SM = 8 warps x MINB x 32
// lanes x UU x 32 B): how the L2 gather rate grows with the bytes in flight (latency- vs bandwidth-bound)
template <int UU, int MINB>
__global__ void __launch_bounds__(256, MINB) k_probe_u(const char *__restrict__ B, uint32_t nrows, int RB, int iters,
                                                     float *out, unsigned long long *cyc) {
    const int lane = threadIdx.x & 31;
    const uint64_t wid = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    float acc = 0.f;
    const long long t0 = clock64();
    const int g = lane / 8, gl = lane % 8;
    for (int it = 0; it < iters; ++it) {
        f8 x[UU];
#pragma unroll
        for (int u = 0; u < UU; ++u) {
            const uint32_t r = hrow(((wid * iters + it) * UU + u) * 8 + g, nrows);
            x[u] = ld8<false>(B + (size_t)r * RB + (size_t)((it * UU + u) & (RB / 256 - 1)) * 256 + gl * 32);
        }
#pragma unroll
        for (int u = 0; u < UU; ++u) acc += x[u].lo.x + x[u].hi.w;
    }
    const long long t1 = clock64();
    out[(uint64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
    if (threadIdx.x == 0) atomicMax(cyc + blockIdx.x % 1024, (unsigned long long)(t1 - t0));
}

// Mixed residency (C5-like): a fraction far_pct of the row gathers go to a 1 GB window (DRAM misses), the rest to a
// small L2-resident window; PF: each lane also issues prefetch.global.L2 for its sector of the rows it will load
// PFD iterations later (a register-free way to bring far rows into L2 ahead of the register loads).
template <int UU, int PF>
__global__ void __launch_bounds__(256, 3) k_probe_mix(const char *__restrict__ B, uint32_t near_rows, uint32_t far_rows,
                                                      int far_pct, int RB, int iters, float *out,
                                                      unsigned long long *cyc) {
    const int lane = threadIdx.x & 31;
    const uint64_t wid = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int g = lane / 8, gl = lane % 8;
    float acc = 0.f;
    const long long t0 = clock64();
    auto addr = [&](uint64_t q) -> const char * {
        const uint32_t hsh = (uint32_t)q * 0x9E3779B1u;
        const bool far = (hsh >> 25) % 100u < (uint32_t)far_pct;
        const uint32_t r = far ? (((hsh * 0x85EBCA6Bu) >> 3) & (far_rows - 1)) + near_rows : (hsh >> 7) & (near_rows - 1);
        return B + (size_t)r * RB;
    };
    for (int it = 0; it < iters; ++it) {
        if (PF > 0) {
#pragma unroll
            for (int u = 0; u < UU; ++u) {
                const char *p = addr(((wid * iters + it + PF) * UU + u) * 8 + g) + gl * 32;
                asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
            }
        }
        f8 x[UU];
#pragma unroll
        for (int u = 0; u < UU; ++u) x[u] = ld8<false>(addr(((wid * iters + it) * UU + u) * 8 + g) + gl * 32);
#pragma unroll
        for (int u = 0; u < UU; ++u) acc += x[u].lo.x + x[u].hi.w;
    }
    const long long t1 = clock64();
    out[(uint64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
    if (threadIdx.x == 0) atomicMax(cyc + blockIdx.x % 1024, (unsigned long long)(t1 - t0));
}

// shape 5: rows staged in shared memory (window <= 192 KB), gathered with LDS.128 (warp per 512-B row)
__global__ void __launch_bounds__(256, 1) k_probe_smem(const char *__restrict__ B, uint32_t nrows, int RB, int iters,
                                                       float *out, unsigned long long *cyc) {
    extern __shared__ __align__(16) char sm[];
    for (uint32_t i = threadIdx.x; i < nrows * RB / 16; i += blockDim.x)
        reinterpret_cast<float4 *>(sm)[i] = reinterpret_cast<const float4 *>(B)[i];
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const uint64_t wid = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    float acc = 0.f;
    const long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        float4 x[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t r = hrow((wid * iters + it) * U + u, nrows);
            x[u] = reinterpret_cast<const float4 *>(sm + (size_t)r * RB)[((it * U + u) & (RB / 512 - 1)) * 32 + lane];
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc += x[u].x + x[u].w;
    }
    const long long t1 = clock64();
    out[(uint64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
    if (threadIdx.x == 0) atomicMax(cyc + blockIdx.x % 1024, (unsigned long long)(t1 - t0));
}

// Library entry (tools/__init__.py ldpath_gather): best of `reps` launches of one shape over one window;
// returns GB/s (-1 on error) and the bytes per SM clock in *bpc.
extern "C" double ldpath_gather(int shape, int64_t window, int RB, int reps, double *bpc) {
    int sms = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    char *B = nullptr;
    float *out = nullptr;
    unsigned long long *cyc = nullptr;
    if (cudaMalloc(&B, (size_t)window) != cudaSuccess) return -1.0;
    cudaMemset(B, 0, (size_t)window);
    cudaMalloc(&out, (size_t)sms * 3 * 256 * sizeof(float));
    cudaMalloc(&cyc, 1024 * sizeof(unsigned long long));
    const uint32_t nrows = (uint32_t)(window / RB);
    const int blocks = sms * 3, iters = 512;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    double best = -1.0, best_bpc = 0.0;
    for (int rep = 0; rep < reps; ++rep) {
        cudaMemset(cyc, 0, 1024 * sizeof(unsigned long long));
        cudaEventRecord(e0);
        switch (shape) {
            case 0: k_probe<0><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
            case 3: k_probe<3><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
            default: k_probe<1><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
        }
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        unsigned long long hc[1024];
        cudaMemcpy(hc, cyc, sizeof(hc), cudaMemcpyDeviceToHost);
        unsigned long long mc = 1;
        for (int i = 0; i < 1024; ++i) mc = hc[i] > mc ? hc[i] : mc;
        const double per_instr = (shape == 0 || shape == 3) ? 1024.0 : 512.0;
        const double bytes = (double)blocks * 8 * iters * U * per_instr;
        const double gbs = bytes / (ms * 1e-3) / 1e9;
        if (gbs > best) { best = gbs; best_bpc = bytes / sms / (double)mc; }
    }
    if (cudaGetLastError() != cudaSuccess) best = -1.0;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(B);
    cudaFree(out);
    cudaFree(cyc);
    if (bpc) *bpc = best_bpc;
    return best;
}

#ifndef LDPATH_NO_MAIN
// ./ldpathprobe sweep: shape 0 (k_spmm's) over windows x row sizes
static int sweep() {
    printf("{\"sweep\": [\n");
    bool first = true;
    for (int64_t wmb : {1, 4, 16, 32, 64, 100}) {
        for (int rb : {256, 512, 1024, 2048}) {
            double bpc = 0;
            const double gbs = ldpath_gather(0, wmb << 20, rb, 5, &bpc);
            printf("%s{\"window_mb\": %lld, \"row_bytes\": %d, \"GBps\": %.1f, \"bytes_per_sm_clk\": %.2f}",
                   first ? "" : ",\n", (long long)wmb, rb, gbs, bpc);
            first = false;
        }
    }
    printf("\n]}\n");
    return 0;
}

template <int UU, int MINB>
static void run_u(const char *B, int64_t window, int RB, int sms, float *out, unsigned long long *cyc, bool &first) {
    const uint32_t nrows = (uint32_t)(window / RB);
    const int blocks = sms * MINB, iters = 2048 / UU;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    double best = 0, best_bpc = 0;
    for (int rep = 0; rep < 5; ++rep) {
        cudaMemset(cyc, 0, 1024 * sizeof(unsigned long long));
        cudaEventRecord(e0);
        k_probe_u<UU, MINB><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        unsigned long long hc[1024];
        cudaMemcpy(hc, cyc, sizeof(hc), cudaMemcpyDeviceToHost);
        unsigned long long mc = 1;
        for (int i = 0; i < 1024; ++i) mc = hc[i] > mc ? hc[i] : mc;
        const double bytes = (double)blocks * 8 * iters * UU * 1024.0;
        const double gbs = bytes / (ms * 1e-3) / 1e9;
        if (gbs > best) { best = gbs; best_bpc = bytes / sms / (double)mc; }
    }
    printf("%s{\"window_mb\": %lld, \"U\": %d, \"ctas_per_sm\": %d, \"inflight_kb_per_sm\": %d, \"GBps\": %.1f, "
           "\"bytes_per_sm_clk\": %.2f, \"err\": \"%s\"}", first ? "" : ",\n", (long long)(window >> 20), UU, MINB,
           8 * MINB * 32 * UU * 32 / 1024, best, best_bpc, cudaGetErrorString(cudaGetLastError()));
    first = false;
}

static int inflight() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    char *B;
    float *out;
    unsigned long long *cyc;
    cudaMalloc(&B, (size_t)1 << 30);
    cudaMemset(B, 0, (size_t)1 << 30);
    cudaMalloc(&out, (size_t)sms * 8 * 256 * sizeof(float));
    cudaMalloc(&cyc, 1024 * sizeof(unsigned long long));
    printf("{\"inflight\": [\n");
    bool first = true;
    for (int64_t wmb : {16, 100, 1024}) {
        const int64_t w = wmb << 20;
        run_u<1, 3>(B, w, 512, sms, out, cyc, first);
        run_u<2, 3>(B, w, 512, sms, out, cyc, first);
        run_u<4, 3>(B, w, 512, sms, out, cyc, first);
        run_u<4, 2>(B, w, 512, sms, out, cyc, first);
        run_u<8, 2>(B, w, 512, sms, out, cyc, first);
        run_u<8, 1>(B, w, 512, sms, out, cyc, first);
        run_u<16, 1>(B, w, 512, sms, out, cyc, first);
        run_u<2, 4>(B, w, 512, sms, out, cyc, first);
        run_u<4, 4>(B, w, 512, sms, out, cyc, first);
    }
    printf("\n]}\n");
    return 0;
}

template <int UU, int PF>
static void run_mix(const char *B, int far_pct, int sms, float *out, unsigned long long *cyc, bool &first) {
    const int RB = 256;                                  // one group load = one 256-B row slice
    const uint32_t near_rows = (4u << 20) / RB, far_rows = (512u << 20) / RB;   // 4 MB near (L2), 512 MB far
    const int blocks = sms * 3, iters = 2048 / UU;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    double best = 0;
    for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(e0);
        k_probe_mix<UU, PF><<<blocks, 256>>>(B, near_rows, far_rows, far_pct, RB, iters, out, cyc);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        const double bytes = (double)blocks * 8 * iters * UU * 1024.0;
        best = std::max(best, bytes / (ms * 1e-3) / 1e9);
    }
    printf("%s{\"far_pct\": %d, \"U\": %d, \"prefetch_ahead\": %d, \"GBps\": %.1f, \"err\": \"%s\"}",
           first ? "" : ",\n", far_pct, UU, PF, best, cudaGetErrorString(cudaGetLastError()));
    first = false;
}

static int mixed() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    char *B;
    float *out;
    unsigned long long *cyc;
    cudaMalloc(&B, (size_t)1 << 30);
    cudaMemset(B, 0, (size_t)1 << 30);
    cudaMalloc(&out, (size_t)sms * 3 * 256 * sizeof(float));
    cudaMalloc(&cyc, 1024 * sizeof(unsigned long long));
    printf("{\"mixed\": [\n");
    bool first = true;
    for (int fp : {0, 10, 20, 40, 100}) {
        run_mix<4, 0>(B, fp, sms, out, cyc, first);
        run_mix<4, 1>(B, fp, sms, out, cyc, first);
        run_mix<4, 2>(B, fp, sms, out, cyc, first);
        run_mix<4, 4>(B, fp, sms, out, cyc, first);
        run_mix<2, 0>(B, fp, sms, out, cyc, first);
        run_mix<2, 2>(B, fp, sms, out, cyc, first);
    }
    printf("\n]}\n");
    return 0;
}

int main(int argc, char **argv) {
    if (argc > 1 && argv[1][0] == 's') return sweep();
    if (argc > 1 && argv[1][0] == 'i') return inflight();
    if (argc > 1 && argv[1][0] == 'm') return mixed();
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int RB = argc > 1 ? atoi(argv[1]) : 512;   // a power of two >= 512
    const size_t Bbytes = (size_t)1 << 30;
    char *B;
    float *out;
    unsigned long long *cyc;
    cudaMalloc(&B, Bbytes);
    cudaMemset(B, 0, Bbytes);
    cudaMalloc(&out, (size_t)sms * 3 * 256 * sizeof(float));
    cudaMalloc(&cyc, 1024 * sizeof(unsigned long long));
    cudaFuncSetAttribute(k_probe_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    const size_t windows[] = {32u << 10, 160u << 10, 16u << 20, 1u << 30};
    const char *wname[] = {"32KB(L1)", "160KB(L1)", "16MB(L2)", "1GB(HBM)"};
    const int iters = 512;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    printf("{\"row_bytes\": %d, \"sms\": %d, \"results\": [\n", RB, sms);
    bool first = true;
    for (int shape = 0; shape <= 5; ++shape) {
        for (int wi = 0; wi < 4; ++wi) {
            if (shape == 5 && wi > 1) continue;
            const uint32_t nrows = (uint32_t)(windows[wi] / RB);
            const int blocks = shape == 5 ? sms : sms * 3;
            double best_gbs = 0, best_bpc = 0;
            for (int rep = 0; rep < 5; ++rep) {
                cudaMemset(cyc, 0, 1024 * sizeof(unsigned long long));
                cudaEventRecord(e0);
                switch (shape) {
                    case 0: k_probe<0><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
                    case 1: k_probe<1><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
                    case 2: k_probe<2><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
                    case 3: k_probe<3><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
                    case 4: k_probe<4><<<blocks, 256>>>(B, nrows, RB, iters, out, cyc); break;
                    default: k_probe_smem<<<blocks, 256, (size_t)nrows * RB>>>(B, nrows, RB, iters, out, cyc); break;
                }
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                float ms = 0;
                cudaEventElapsedTime(&ms, e0, e1);
                unsigned long long hc[1024];
                cudaMemcpy(hc, cyc, sizeof(hc), cudaMemcpyDeviceToHost);
                unsigned long long mc = 0;
                for (int i = 0; i < 1024; ++i) mc = hc[i] > mc ? hc[i] : mc;
                // bytes per warp instruction x instructions
                const double per_instr = shape == 0 || shape == 3 || shape == 4 ? 1024.0 : shape == 2 ? 128.0 : 512.0;
                const double bytes = (double)blocks * 8 * iters * U * per_instr;
                const double gbs = bytes / (ms * 1e-3) / 1e9;
                const double bpc = bytes / sms / (double)mc;     // bytes per SM per SM-clock (timed loop only)
                if (gbs > best_gbs) { best_gbs = gbs; best_bpc = bpc; }
            }
            cudaError_t err = cudaGetLastError();
            printf("%s{\"shape\": %d, \"window\": \"%s\", \"GBps\": %.1f, \"bytes_per_sm_clk\": %.2f, \"err\": \"%s\"}",
                   first ? "" : ",\n", shape, wname[wi], best_gbs, best_bpc, cudaGetErrorString(err));
            first = false;
        }
    }
    printf("\n]}\n");
    return 0;
}
#endif
