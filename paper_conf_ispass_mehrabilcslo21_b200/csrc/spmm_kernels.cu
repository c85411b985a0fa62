// spmm_kernels.cu -- the timed SpMM of the hot path (a8):
//   C[perm[p]][k] = sum_{j in row' p} value'[j] * B[colidx'[j]][k]      (Alg.1)
// on the row-permuted CSR, with the inverse permutation fused into the C store.
//
// B200 design (DESIGN.md §"SpMM kernel"), not the paper's warp-per-row Volta kernel:
//   * a row is owned by a lane GROUP of G lanes; each lane owns V float4 column vectors of the C
//     row (4*V*G columns per tile), so a warp works on 32/G consecutive permuted rows at once and
//     the sorted/clustered orders decide how balanced those rows are (the paper's "warp load",
//     P:L84-88, re-expressed for this mapping);
//   * per nnz, the G lanes of a group broadcast-load the interleaved (col, val) pair (8 B) and issue
//     V coalesced 16-byte loads of the B row (G*16 B contiguous per vector), then 4*V FP32 FMAs as
//     packed FFMA2 (sm_100 fma.rn.f32x2) -- every accumulator is a sequential chain in ascending j,
//     the order of the oracle's definition (oracle.c c1);
//   * rows longer than split_nnz are cut into split_nnz-nnz chunks processed like rows; their
//     partial sums are combined in a fixed pairwise order by k_combine (deterministic, bounded
//     rounding, DESIGN.md §"Accuracy");
//   * C is written once with streaming stores at C[perm[p]] (original order, beta = 0).
// Bound: HBM bandwidth (algorithmic bytes 4(M+1) + 8 nnz + 4K|cols(A)| + 4MK, BASELINE.json north star).
#include "internal.cuh"
#include <algorithm>

namespace spmm {
namespace {

constexpr int SPMM_THREADS = 256;

__device__ __forceinline__ void fma4(float a, const float4 &b, float4 &acc) {
    float2 lo = __ffma2_rn(make_float2(a, a), make_float2(b.x, b.y), make_float2(acc.x, acc.y));
    float2 hi = __ffma2_rn(make_float2(a, a), make_float2(b.z, b.w), make_float2(acc.z, acc.w));
    acc.x = lo.x; acc.y = lo.y; acc.z = hi.x; acc.w = hi.y;
}

// U nnz per iteration, V float4 per lane, G lanes per row, MASK: column tail present.
template <int V, int G, bool MASK>
__global__ void __launch_bounds__(SPMM_THREADS) k_spmm(const int32_t *__restrict__ rowptr, const int2 *__restrict__ cv,
                                                       const int32_t *__restrict__ perm, const float4 *__restrict__ B4,
                                                       float4 *__restrict__ C4, int64_t M, int32_t K4, int32_t split,
                                                       const int32_t *__restrict__ cstart,
                                                       const int32_t *__restrict__ clen, int64_t n_chunks,
                                                       float4 *__restrict__ P4) {
    constexpr int RPW = 32 / G;
    constexpr int CT4 = V * G;
    constexpr int U = 2;
    const int lane = threadIdx.x & 31;
    const int g = lane / G, gl = lane % G;
    const int col0 = blockIdx.y * CT4 + gl;      // this lane's first float4 column; then + v*G
    const int64_t row_tasks = (M + RPW - 1) / RPW;
    const int64_t total = row_tasks + (n_chunks + RPW - 1) / RPW;
    const int64_t nwarps = (int64_t)gridDim.x * (SPMM_THREADS / 32);
    bool colok[V];
#pragma unroll
    for (int v = 0; v < V; ++v) colok[v] = !MASK || (col0 + v * G < K4);

    for (int64_t t = (int64_t)blockIdx.x * (SPMM_THREADS / 32) + (threadIdx.x >> 5); t < total; t += nwarps) {
        int32_t start = 0, end = 0;
        float4 *dst = nullptr;
        if (t < row_tasks) {
            const int64_t p = t * RPW + g;
            if (p < M) {
                start = __ldg(rowptr + p);
                end = __ldg(rowptr + p + 1);
                if (end - start <= split) dst = C4 + (size_t)__ldg(perm + p) * K4;
            }
        } else {
            const int64_t c = (t - row_tasks) * RPW + g;
            if (c < n_chunks) {
                start = __ldg(cstart + c);
                end = start + __ldg(clen + c);
                dst = P4 + (size_t)c * K4;
            }
        }
        if (dst == nullptr) continue;   // long row (its chunks do the work) or past the end
        float4 acc[V];
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = make_float4(0.f, 0.f, 0.f, 0.f);
        int32_t j = start;
        for (; j + U <= end; j += U) {
            int2 e[U];
#pragma unroll
            for (int u = 0; u < U; ++u) e[u] = __ldg(cv + j + u);
            float4 x[U][V];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const float4 *b = B4 + (size_t)e[u].x * K4 + col0;
#pragma unroll
                for (int v = 0; v < V; ++v) x[u][v] = colok[v] ? __ldg(b + v * G) : make_float4(0.f, 0.f, 0.f, 0.f);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const float a = __int_as_float(e[u].y);
#pragma unroll
                for (int v = 0; v < V; ++v) fma4(a, x[u][v], acc[v]);
            }
        }
        if (j < end) {
            const int2 e = __ldg(cv + j);
            const float4 *b = B4 + (size_t)e.x * K4 + col0;
            const float a = __int_as_float(e.y);
#pragma unroll
            for (int v = 0; v < V; ++v)
                if (colok[v]) fma4(a, __ldg(b + v * G), acc[v]);
        }
#pragma unroll
        for (int v = 0; v < V; ++v)
            if (colok[v]) __stcs(dst + col0 + v * G, acc[v]);
    }
}

// Pairwise (binary-counter) combine of a long row's chunk partials, fixed order -> deterministic;
// rounding grows with log2(#chunks) instead of #chunks.  One CTA per long row, thread per float4.
__global__ void __launch_bounds__(128) k_combine(const float4 *__restrict__ P4, const int32_t *__restrict__ long_pos,
                                                 const int32_t *__restrict__ long_chunk_ptr,
                                                 const int32_t *__restrict__ perm, float4 *__restrict__ C4,
                                                 int32_t K4) {
    const int32_t l = blockIdx.x;
    const int32_t c0 = long_chunk_ptr[l], c1 = long_chunk_ptr[l + 1];
    float4 *dst = C4 + (size_t)perm[long_pos[l]] * K4;
    for (int32_t col = threadIdx.x; col < K4; col += blockDim.x) {
        float4 stk[32];
        int sp = 0;
        for (int32_t i = 0; i < c1 - c0; ++i) {
            float4 x = P4[(size_t)(c0 + i) * K4 + col];
            for (uint32_t cnt = (uint32_t)i + 1u; (cnt & 1u) == 0u; cnt >>= 1) {
                const float4 y = stk[--sp];
                x = make_float4(y.x + x.x, y.y + x.y, y.z + x.z, y.w + x.w);
            }
            stk[sp++] = x;
        }
        float4 r = stk[--sp];
        while (sp > 0) {
            const float4 y = stk[--sp];
            r = make_float4(y.x + r.x, y.y + r.y, y.z + r.z, y.w + r.w);
        }
        __stcs(dst + col, r);
    }
}

__global__ void k_zero_rows(float4 *C4, int64_t n4) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x)
        C4[i] = make_float4(0.f, 0.f, 0.f, 0.f);
}

using SpmmKernel = void (*)(const int32_t *, const int2 *, const int32_t *, const float4 *, float4 *, int64_t, int32_t,
                            int32_t, const int32_t *, const int32_t *, int64_t, float4 *);

template <int V, bool MASK>
SpmmKernel pick_g(int G) {
    switch (G) {
        case 1: return k_spmm<V, 1, MASK>;
        case 2: return k_spmm<V, 2, MASK>;
        case 4: return k_spmm<V, 4, MASK>;
        case 8: return k_spmm<V, 8, MASK>;
        case 16: return k_spmm<V, 16, MASK>;
        default: return k_spmm<V, 32, MASK>;
    }
}

struct Config {
    SpmmKernel kern;
    int V, G, tiles;
};

// exact fit 4*V*G == K with V in {4,3,2,1}, G a power of two <= 32; else V=4 with a masked tail
Config choose(int32_t K4) {
    for (int V = 4; V >= 1; --V) {
        if (K4 % V) continue;
        int G = K4 / V;
        if (G >= 1 && G <= 32 && (G & (G - 1)) == 0) {
            SpmmKernel k = V == 4 ? pick_g<4, false>(G) : V == 3 ? pick_g<3, false>(G) : V == 2 ? pick_g<2, false>(G)
                                                                                            : pick_g<1, false>(G);
            return {k, V, G, 1};
        }
    }
    int G = 1;
    while (G < 32 && 4 * G < K4) G <<= 1;
    int tiles = (int)ceil_div(K4, 4 * G);
    return {pick_g<4, true>(G), 4, G, tiles};
}

}  // namespace

spmm_status launch_spmm(spmm_ctx *h, const float *B, int64_t K, float *C, cudaStream_t s, int32_t *launches) {
    *launches = 0;
    const int64_t M = h->M;
    if (M == 0) return SPMM_OK;
    const int32_t K4 = (int32_t)(K / 4);
    if (h->nnz == 0) {
        k_zero_rows<<<(unsigned)std::min<int64_t>(ceil_div(M * K4, 256), 148 * 16), 256, 0, s>>>(
            reinterpret_cast<float4 *>(C), M * K4);
        SPMM_CUDA(cudaGetLastError());
        *launches = 1;
        return SPMM_OK;
    }
    const LongRows &lr = h->lr;
    float4 *P4 = nullptr;
    if (lr.n_chunks > 0) {
        size_t need = (size_t)lr.n_chunks * K * sizeof(float);
        if (h->partials.bytes < need) SPMM_TRY(h->partials.alloc(need, s));
        P4 = h->partials.as<float4>();
    }
    Config cfg = choose(K4);
    const int rpw = 32 / cfg.G;
    const int64_t tasks = ceil_div(M, rpw) + ceil_div(lr.n_chunks, rpw);
    int occ = 0;
    SPMM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, cfg.kern, SPMM_THREADS, 0));
    occ = std::max(occ, 1);
    const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(tasks, SPMM_THREADS / 32),
                                                                  (int64_t)h->num_sms * occ));
    dim3 grid((unsigned)blocks, (unsigned)cfg.tiles);
    cfg.kern<<<grid, SPMM_THREADS, 0, s>>>(h->rowptr_p.as<int32_t>(), h->cv_p.as<int2>(), h->perm.as<int32_t>(),
                                           reinterpret_cast<const float4 *>(B), reinterpret_cast<float4 *>(C), M, K4,
                                           h->params.split_nnz, lr.chunk_start.as<int32_t>(), lr.chunk_len.as<int32_t>(),
                                           lr.n_chunks, P4);
    SPMM_CUDA(cudaGetLastError());
    *launches = 1;
    if (lr.n_long > 0) {
        k_combine<<<(unsigned)lr.n_long, 128, 0, s>>>(P4, lr.long_pos.as<int32_t>(), lr.long_chunk_ptr.as<int32_t>(),
                                                     h->perm.as<int32_t>(), reinterpret_cast<float4 *>(C), K4);
        SPMM_CUDA(cudaGetLastError());
        *launches = 2;
    }
    return SPMM_OK;
}

}  // namespace spmm
