// spmm_kernels.cu -- the timed SpMM of the hot path (a8):
//   C[perm[p]][k] = sum_{j in row' p} value'[j] * B[colidx'[j]][k]      (Alg.1)
// on the row-permuted CSR, with the inverse permutation fused into the C store, plus the a7 run
// schedule (row classes: empty / whole / split rows) it executes.
//
// B200 design (DESIGN.md §"SpMM kernel"), not the paper's warp-per-row Volta kernel:
//   * a work unit is owned by a lane GROUP of G lanes; each lane owns V float4 column vectors of the
//     C row (4*V*G columns per tile), so a warp works on RPW = 32/G units at once, and the sorted /
//     clustered orders decide how balanced those units are (the paper's "warp load", P:L84-88,
//     re-expressed for this mapping);
//   * per nnz, the G lanes of a group broadcast-load the interleaved (col, val) pair (8 B) and issue
//     V coalesced 16-byte loads of the B row (G*16 B contiguous per vector), then 4*V FP32 FMAs as
//     packed FFMA2 (sm_100 fma.rn.f32x2) -- every accumulator is a sequential chain in ascending j,
//     the order of the oracle's definition (oracle.c c1);
//   * warp tasks follow the permuted order: runs of non-empty short rows are packed RPW per task;
//     a row longer than split_nnz is cut into split_nnz-nnz chunks, RPW consecutive chunks form one
//     warp task whose group sums are reduced across the warp in a fixed butterfly tree, and the
//     per-task partials are combined in a fixed pairwise order by k_combine (deterministic, bounded
//     rounding, DESIGN.md §"Accuracy"); all chunking is relative to the row start, so C is
//     bit-identical for every permutation;
//   * empty rows are a class of their own (zero-filled, the B200 form of DCSR's skip);
//   * C is written once with streaming stores at C[perm[p]] (original order, beta = 0).
// Bound: HBM bandwidth (algorithmic bytes 4(M+1) + 8 nnz + 4K|cols(A)| + 4MK, BASELINE.json north star).
#include "internal.cuh"
#include <algorithm>
#include <climits>
#include <cstdlib>

namespace spmm {
namespace {

constexpr int SPMM_THREADS = 256;
constexpr int32_t NOSTORE = INT_MIN;

__device__ __forceinline__ void fma4(float a, const float4 &b, float4 &acc) {
    float2 lo = __ffma2_rn(make_float2(a, a), make_float2(b.x, b.y), make_float2(acc.x, acc.y));
    float2 hi = __ffma2_rn(make_float2(a, a), make_float2(b.z, b.w), make_float2(acc.z, acc.w));
    acc.x = lo.x; acc.y = lo.y; acc.z = hi.x; acc.w = hi.y;
}

// L2 cache-policy loads (VAR & 1): B rows are the reused operand -> L2::evict_last; the streamed
// (col, val) pairs -> L2::evict_first and no L1 allocation.
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
template <bool HINT>
__device__ __forceinline__ float4 ld_b(const float4 *ptr, uint64_t pol) {
    if (!HINT) return __ldg(ptr);
    float4 r;
    asm("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
        : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(ptr), "l"(pol));
    return r;
}
template <bool HINT>
__device__ __forceinline__ int2 ld_cv(const int2 *ptr, uint64_t pol) {
    if (!HINT) return __ldg(ptr);
    int2 r;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.s32 {%0,%1}, [%2], %3;" : "=r"(r.x), "=r"(r.y) : "l"(ptr), "l"(pol));
    return r;
}

// V float4 per lane, G lanes per unit, MASK: column tail present (K not a multiple of 4*V*G).
// VAR bit 0: L2 cache-policy hints; bit 1: U = 4 nnz per step for V = 4.
// Warp tasks are claimed dynamically (one atomicAdd per task on a per-column-tile counter), so the set
// of tasks in flight stays a narrow window of the permuted order whatever the task costs: the order's
// B-row locality survives into L2 and no warp is left with a long static tail.
// CTA-contiguous task claiming (SCHED = 1): the CTA takes chunks of CTA_CHUNK consecutive warp tasks
// from the global counter, so the consecutive rows of a chunk run concurrently on one SM (the paper's
// "clusters of N_w consecutive rows ... processed in parallel" by a CTA) and their shared B rows
// can hit in L1.  Warps draw tickets from a shared-memory counter; ticket k belongs to local chunk
// k / CTA_CHUNK, whose global id is published in a ring slot by the warp holding its first ticket.  A
// slot is republished only after all readers of its previous chunk have read it (no ABA, no barrier).
constexpr int CTA_CHUNK = SPMM_THREADS / 32;
constexpr int RING = 4;

struct TaskQueue {
    unsigned int ticket;
    unsigned int gid[RING];
    int tag[RING];
    int pending[RING];
};

__device__ __forceinline__ unsigned int claim_task(TaskQueue *q, unsigned int *gcounter, int lane) {
    unsigned int task = 0;
    if (lane == 0) {
        const unsigned int k = atomicAdd(&q->ticket, 1u);
        const int c = (int)(k / CTA_CHUNK), w = (int)(k % CTA_CHUNK), s = c % RING;
        volatile int *vtag = q->tag;
        volatile int *vpend = q->pending;
        volatile unsigned int *vgid = q->gid;
        unsigned int g;
        if (w == 0) {
            while (vpend[s] != 0) { }
            g = atomicAdd(gcounter, 1u);
            vgid[s] = g;
            vpend[s] = CTA_CHUNK - 1;
            __threadfence_block();
            vtag[s] = c;
        } else {
            while (vtag[s] != c) { }
            __threadfence_block();
            g = vgid[s];
            atomicSub(&q->pending[s], 1);
        }
        task = g * CTA_CHUNK + (unsigned int)w;
    }
    return __shfl_sync(0xffffffffu, task, 0);
}

template <int V, int G, bool MASK, int SCHED, int VAR>
__global__ void __launch_bounds__(SPMM_THREADS, 3) k_spmm(const int4 *__restrict__ units, int64_t n_tasks,
                                                       const int2 *__restrict__ cv, const float4 *__restrict__ B4,
                                                       float4 *__restrict__ C4, int32_t K4, float4 *__restrict__ P4,
                                                       unsigned int *__restrict__ counter) {
    constexpr int RPW = 32 / G;
    constexpr int CT4 = V * G;
    constexpr bool HINT = (VAR & 1) != 0;
    constexpr int U = (V >= 3 && !(VAR & 2)) ? 2 : 4;   // nnz per inner step (B loads in flight per lane: U*V)
    constexpr int BATCH = G >= 8 ? G : 8;        // (col, val) pairs prefetched per group per batch
    constexpr int PL = BATCH / G;                // pairs held per lane
    const int lane = threadIdx.x & 31;
    const int g = lane / G, gl = lane % G;
    const int col0 = blockIdx.y * CT4 + gl;      // this lane's first float4 column; then + v*G
    bool colok[V];
#pragma unroll
    for (int v = 0; v < V; ++v) colok[v] = !MASK || (col0 + v * G < K4);
    const uint64_t pol_b = HINT ? policy_evict_last() : 0, pol_a = HINT ? policy_evict_first() : 0;

    __shared__ TaskQueue q;
    unsigned int tk = 0;
    if (SCHED == 1) {
        if (threadIdx.x == 0) {
            q.ticket = 0;
            for (int r = 0; r < RING; ++r) { q.tag[r] = -1; q.pending[r] = 0; q.gid[r] = 0; }
        }
        __syncthreads();
        tk = claim_task(&q, counter + blockIdx.y, lane);
    } else {
        if (lane == 0) tk = atomicAdd(counter + blockIdx.y, 1u);
        tk = __shfl_sync(0xffffffffu, tk, 0);
    }
    int64_t t = tk;
    int4 u = t < n_tasks ? __ldg(units + t * RPW + g) : make_int4(0, 0, NOSTORE, 0);
    while (t < n_tasks) {
        // claim and fetch the next task first, so its latency hides behind this one
        int64_t t_next;
        if (SCHED == 1) {
            t_next = claim_task(&q, counter + blockIdx.y, lane);
        } else {
            if (lane == 0) tk = atomicAdd(counter + blockIdx.y, 1u);
            t_next = __shfl_sync(0xffffffffu, tk, 0);
        }
        const int4 u_next = t_next < n_tasks ? __ldg(units + t_next * RPW + g) : make_int4(0, 0, NOSTORE, 0);
        const int32_t start = u.x, len = u.y, dst = u.z;
        // warp-uniform trip count (groups past their own length are predicated off, not diverged, so
        // the (col, val) shuffles below stay warp-wide)
        const int32_t maxlen = (int32_t)__reduce_max_sync(0xffffffffu, (unsigned)len);
        float4 acc[V];
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = make_float4(0.f, 0.f, 0.f, 0.f);
        // (col, val) pairs: each lane loads PL of the group's next BATCH pairs (coalesced), one batch
        // ahead of use; every nnz is then broadcast inside the group with two shuffles
        int2 cur[PL];
#pragma unroll
        for (int p = 0; p < PL; ++p) {
            const int32_t o = p * G + gl;
            cur[p] = o < len ? ld_cv<HINT>(cv + start + o, pol_a) : make_int2(0, 0);
        }
        for (int32_t b0 = 0; b0 < maxlen; b0 += BATCH) {
            int2 nxt[PL];
#pragma unroll
            for (int p = 0; p < PL; ++p) {
                const int32_t o = b0 + BATCH + p * G + gl;
                nxt[p] = o < len ? ld_cv<HINT>(cv + start + o, pol_a) : make_int2(0, 0);
            }
#pragma unroll
            for (int q0 = 0; q0 < BATCH; q0 += U) {
                int32_t col[U];
                float a[U];
#pragma unroll
                for (int w = 0; w < U; ++w) {
                    const int qq = q0 + w;
                    const int src = g * G + (qq % G);
                    col[w] = __shfl_sync(0xffffffffu, cur[qq / G].x, src);
                    a[w] = __int_as_float(__shfl_sync(0xffffffffu, cur[qq / G].y, src));
                }
                const int32_t rem = len - (b0 + q0);    // nnz left for this group
                if (rem >= U) {                          // full step: U*V independent B loads in flight
                    float4 x[U][V];
#pragma unroll
                    for (int w = 0; w < U; ++w) {
                        const float4 *b = B4 + (size_t)col[w] * K4 + col0;
#pragma unroll
                        for (int v = 0; v < V; ++v)
                            x[w][v] = colok[v] ? ld_b<HINT>(b + v * G, pol_b) : make_float4(0.f, 0.f, 0.f, 0.f);
                    }
#pragma unroll
                    for (int w = 0; w < U; ++w)
#pragma unroll
                        for (int v = 0; v < V; ++v) fma4(a[w], x[w][v], acc[v]);
                } else if (rem > 0) {                    // the group's tail
#pragma unroll
                    for (int w = 0; w < U - 1; ++w) {
                        if (w < rem) {
                            const float4 *b = B4 + (size_t)col[w] * K4 + col0;
#pragma unroll
                            for (int v = 0; v < V; ++v)
                                if (colok[v]) fma4(a[w], ld_b<HINT>(b + v * G, pol_b), acc[v]);
                        }
                    }
                }
            }
#pragma unroll
            for (int p = 0; p < PL; ++p) cur[p] = nxt[p];
        }
        if (dst >= 0) {                                    // a whole row: C[perm[p]]
#pragma unroll
            for (int v = 0; v < V; ++v)
                if (colok[v]) __stcs(C4 + (size_t)dst * K4 + col0 + v * G, acc[v]);
        } else if (dst != NOSTORE) {                       // chunk group of a long row (warp-uniform)
#pragma unroll
            for (int off = G; off < 32; off <<= 1) {       // fixed butterfly: ((c0+c1)+(c2+c3))...
#pragma unroll
                for (int v = 0; v < V; ++v) {
                    acc[v].x += __shfl_xor_sync(0xffffffffu, acc[v].x, off);
                    acc[v].y += __shfl_xor_sync(0xffffffffu, acc[v].y, off);
                    acc[v].z += __shfl_xor_sync(0xffffffffu, acc[v].z, off);
                    acc[v].w += __shfl_xor_sync(0xffffffffu, acc[v].w, off);
                }
            }
            if (g == 0) {
                const int64_t slot = -(int64_t)dst - 1;
#pragma unroll
                for (int v = 0; v < V; ++v)
                    if (colok[v]) P4[slot * K4 + col0 + v * G] = acc[v];
            }
        }
        t = t_next;
        u = u_next;
    }
}

// ---- kernel mode 2: panel-staged SpMM (schedule: panel.cu) --------------------------------------
// One CTA (16 warps) per SM claims panels of consecutive permuted rows.  Per panel it first copies the
// panel's staged B rows into shared memory with cp.async, then its warps claim the panel's work units
// RPW at a time (shared-memory counter); a nnz whose column was staged (col < 0 in the rewritten cv)
// reads its B row from shared memory, the others from global memory, through one generic load.  Same
// per-row FMA order as the row-group kernel; chunks of long rows write partials (combined pairwise).
constexpr int PS_THREADS = 512;

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(gmem) : "memory");
}

template <int V, int G>
__global__ void __launch_bounds__(PS_THREADS, 1) k_spmm_ps(const int4 *__restrict__ units,
                                                           const int32_t *__restrict__ panel_unit_ptr,
                                                           const int32_t *__restrict__ stage_ptr,
                                                           const int32_t *__restrict__ staged_cols, int64_t n_panels,
                                                           const int2 *__restrict__ cv, const float4 *__restrict__ B4,
                                                           float4 *__restrict__ C4, int32_t K4, float4 *__restrict__ P4,
                                                           unsigned int *__restrict__ counter) {
    extern __shared__ float4 sB[];
    __shared__ unsigned int s_panel, s_next;
    constexpr int RPW = 32 / G;
    constexpr int U = V >= 3 ? 2 : 4;
    constexpr int BATCH = G >= 8 ? G : 8;
    constexpr int PL = BATCH / G;
    const int lane = threadIdx.x & 31;
    const int g = lane / G, gl = lane % G;
    for (;;) {
        if (threadIdx.x == 0) { s_panel = atomicAdd(counter, 1u); s_next = 0u; }
        __syncthreads();
        const unsigned int P = s_panel;
        if (P >= n_panels) break;
        const int32_t s0 = stage_ptr[P], ns = stage_ptr[P + 1] - s0;
        for (int32_t i = threadIdx.x; i < ns * K4; i += PS_THREADS) {
            const int32_t r = i / K4, c = i - r * K4;
            cp_async16(sB + (size_t)r * K4 + c, B4 + (size_t)staged_cols[s0 + r] * K4 + c);
        }
        asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
        __syncthreads();
        const int32_t u0 = panel_unit_ptr[P], nu = panel_unit_ptr[P + 1] - u0;
        for (;;) {
            unsigned int kk = 0;
            if (lane == 0) kk = atomicAdd(&s_next, (unsigned)RPW);
            kk = __shfl_sync(0xffffffffu, kk, 0);
            if ((int32_t)kk >= nu) break;
            const int4 u = (int32_t)kk + g < nu ? __ldg(units + u0 + kk + g) : make_int4(0, 0, NOSTORE, 0);
            const int32_t start = u.x, len = u.y, dst = u.z;
            const int32_t maxlen = (int32_t)__reduce_max_sync(0xffffffffu, (unsigned)len);
            float4 acc[V];
#pragma unroll
            for (int v = 0; v < V; ++v) acc[v] = make_float4(0.f, 0.f, 0.f, 0.f);
            int2 cur[PL];
#pragma unroll
            for (int p = 0; p < PL; ++p) {
                const int32_t o = p * G + gl;
                cur[p] = o < len ? __ldg(cv + start + o) : make_int2(0, 0);
            }
            for (int32_t b0 = 0; b0 < maxlen; b0 += BATCH) {
                int2 nxt[PL];
#pragma unroll
                for (int p = 0; p < PL; ++p) {
                    const int32_t o = b0 + BATCH + p * G + gl;
                    nxt[p] = o < len ? __ldg(cv + start + o) : make_int2(0, 0);
                }
#pragma unroll
                for (int q0 = 0; q0 < BATCH; q0 += U) {
                    int32_t col[U];
                    float a[U];
#pragma unroll
                    for (int w = 0; w < U; ++w) {
                        const int qq = q0 + w;
                        const int src = g * G + (qq % G);
                        col[w] = __shfl_sync(0xffffffffu, cur[qq / G].x, src);
                        a[w] = __int_as_float(__shfl_sync(0xffffffffu, cur[qq / G].y, src));
                    }
                    const int32_t rem = len - (b0 + q0);
                    if (rem >= U) {
                        float4 x[U][V];
#pragma unroll
                        for (int w = 0; w < U; ++w) {
                            const float4 *b = col[w] < 0 ? sB + (size_t)(col[w] & 0x7fffffff) * K4 + gl
                                                         : B4 + (size_t)col[w] * K4 + gl;
#pragma unroll
                            for (int v = 0; v < V; ++v) x[w][v] = b[v * G];
                        }
#pragma unroll
                        for (int w = 0; w < U; ++w)
#pragma unroll
                            for (int v = 0; v < V; ++v) fma4(a[w], x[w][v], acc[v]);
                    } else if (rem > 0) {
#pragma unroll
                        for (int w = 0; w < U - 1; ++w) {
                            if (w < rem) {
                                const float4 *b = col[w] < 0 ? sB + (size_t)(col[w] & 0x7fffffff) * K4 + gl
                                                             : B4 + (size_t)col[w] * K4 + gl;
#pragma unroll
                                for (int v = 0; v < V; ++v) fma4(a[w], b[v * G], acc[v]);
                            }
                        }
                    }
                }
#pragma unroll
                for (int p = 0; p < PL; ++p) cur[p] = nxt[p];
            }
            if (dst >= 0) {
#pragma unroll
                for (int v = 0; v < V; ++v) __stcs(C4 + (size_t)dst * K4 + gl + v * G, acc[v]);
            } else if (dst != NOSTORE) {
                const int64_t slot = -(int64_t)dst - 1;
#pragma unroll
                for (int v = 0; v < V; ++v) P4[slot * K4 + gl + v * G] = acc[v];
            }
        }
        __syncthreads();   // every warp is done with this panel before the next one is staged
    }
}

// Pairwise (binary-counter) combine of a long row's chunk-group partials, fixed order -> deterministic;
// rounding grows with log2(#groups).  One CTA per long row, thread per float4 column.
__global__ void __launch_bounds__(128) k_combine(const float4 *__restrict__ P4, const int32_t *__restrict__ pslot_ptr,
                                                 const int32_t *__restrict__ long_dst, float4 *__restrict__ C4,
                                                 int32_t K4) {
    const int32_t l = blockIdx.x;
    const int32_t c0 = pslot_ptr[l], c1 = pslot_ptr[l + 1];
    float4 *dst = C4 + (size_t)long_dst[l] * K4;
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

// empty rows: zero-fill their C rows (thread per float4)
__global__ void k_zero_rows(const int32_t *__restrict__ rows, int64_t n, int32_t K4, float4 *__restrict__ C4) {
    const int64_t total = n * K4;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
        __stcs(C4 + (size_t)rows[i / K4] * K4 + (i % K4), make_float4(0.f, 0.f, 0.f, 0.f));
}

// ---- a7 schedule construction ------------------------------------------------------------------
// class flags per position: 0 empty, 1 short (0 < len <= split), 2 long
__global__ void k_class_flags(const int32_t *rowptr, int64_t M, int32_t split, int32_t *is_empty, int32_t *is_short,
                              int32_t *is_long) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        const int32_t len = rowptr[p + 1] - rowptr[p];
        is_empty[p] = len == 0;
        is_short[p] = len > 0 && len <= split;
        is_long[p] = len > split;
    }
}

__global__ void k_scatter_flagged(const int32_t *flag, const int32_t *pos, const int32_t *val, int64_t M, int32_t *out) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x)
        if (flag[p]) out[pos[p]] = val ? val[p] : (int32_t)p;
}

// per "segment" k = 0..n_long: the run of short rows before long row k (k = n_long: trailing run) and
// long row k itself.  tasks_k = ceil(s_k / RPW) + ceil(nch_k / RPW); groups_k = ceil(nch_k / RPW).
__global__ void k_segment_counts(const int32_t *lpos, int64_t n_long, const int32_t *sp, int32_t n_short,
                                 const int32_t *rowptr, int32_t split, int32_t rpw, int32_t *tasks, int32_t *groups) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k <= n_long; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t before = k > 0 ? sp[lpos[k - 1]] : 0;
        const int32_t upto = k < n_long ? sp[lpos[k]] : n_short;
        const int32_t s_k = upto - before;
        int32_t nch = 0;
        if (k < n_long) {
            const int32_t len = rowptr[lpos[k] + 1] - rowptr[lpos[k]];
            nch = (len + split - 1) / split;
        }
        const int32_t gk = (nch + rpw - 1) / rpw;
        tasks[k] = (s_k + rpw - 1) / rpw + gk;
        groups[k] = gk;
    }
}

__global__ void k_fill_short(const int32_t *is_short, const int32_t *sp, const int32_t *lidx, const int32_t *lpos,
                             const int32_t *taskbase, const int32_t *rowptr, const int32_t *perm, int64_t M,
                             int32_t rpw, int4 *units) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        if (!is_short[p]) continue;
        const int32_t k = lidx[p];                         // long rows before p = this run's segment
        const int32_t idx = sp[p] - (k > 0 ? sp[lpos[k - 1]] : 0);
        const int64_t task = (int64_t)taskbase[k] + idx / rpw;
        units[task * rpw + idx % rpw] = make_int4(rowptr[p], rowptr[p + 1] - rowptr[p], perm[p], 0);
    }
}

// warp per long row: its chunk groups follow the run of short rows of its segment
__global__ void k_fill_long(const int32_t *lpos, int64_t n_long, const int32_t *sp, const int32_t *taskbase,
                            const int32_t *pslot_ptr, const int32_t *rowptr, const int32_t *perm, int32_t split,
                            int32_t rpw, int4 *units, int32_t *long_dst) {
    const int lane = threadIdx.x & 31;
    for (int64_t k = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < n_long;
         k += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int32_t p = lpos[k];
        const int32_t s_k = sp[p] - (k > 0 ? sp[lpos[k - 1]] : 0);
        const int64_t t0 = (int64_t)taskbase[k] + (s_k + rpw - 1) / rpw;
        const int32_t a = rowptr[p], len = rowptr[p + 1] - a, nch = (len + split - 1) / split;
        const int32_t ng = pslot_ptr[k + 1] - pslot_ptr[k];
        for (int32_t c = lane; c < ng * rpw; c += 32) {
            const int32_t dst = -(pslot_ptr[k] + c / rpw) - 1;
            units[(t0 + c / rpw) * rpw + c % rpw] =
                c < nch ? make_int4(a + c * split, min(split, len - c * split), dst, 0) : make_int4(0, 0, dst, 0);
        }
        if (lane == 0) long_dst[k] = perm[p];
    }
}

__global__ void k_fill_int4(int4 *a, int64_t n, int4 v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) a[i] = v;
}

inline unsigned g1(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 32)); }

spmm_status build_schedule(spmm_ctx *h, int32_t rpw, cudaStream_t s) {
    Schedule &S = h->sched;
    S.rpw = 0;
    const int64_t M = h->M;
    const int32_t split = h->params.split_nnz;
    const int32_t *rowptr = h->rowptr_p.as<int32_t>();
    DevBuf fe, fs, fl, pe, ps, pl, lpos, tasks, groups, taskbase;
    SPMM_TRY(fe.alloc(M * sizeof(int32_t), s));
    SPMM_TRY(fs.alloc(M * sizeof(int32_t), s));
    SPMM_TRY(fl.alloc(M * sizeof(int32_t), s));
    SPMM_TRY(pe.alloc((M + 1) * sizeof(int32_t), s));
    SPMM_TRY(ps.alloc((M + 1) * sizeof(int32_t), s));
    SPMM_TRY(pl.alloc((M + 1) * sizeof(int32_t), s));
    k_class_flags<<<g1(M), 256, 0, s>>>(rowptr, M, split, fe.as<int32_t>(), fs.as<int32_t>(), fl.as<int32_t>());
    SPMM_CUDA(cudaGetLastError());
    int32_t n_empty = 0, n_short = 0, n_long = 0;
    SPMM_TRY(exclusive_scan_i32(fe.as<int32_t>(), pe.as<int32_t>(), M, &n_empty, s));
    SPMM_TRY(exclusive_scan_i32(fs.as<int32_t>(), ps.as<int32_t>(), M, &n_short, s));
    SPMM_TRY(exclusive_scan_i32(fl.as<int32_t>(), pl.as<int32_t>(), M, &n_long, s));
    // empty rows -> their C rows
    S.n_empty = n_empty;
    SPMM_TRY(S.empty_dst.alloc(std::max(n_empty, 1) * sizeof(int32_t), s));
    k_scatter_flagged<<<g1(M), 256, 0, s>>>(fe.as<int32_t>(), pe.as<int32_t>(), h->perm.as<int32_t>(), M,
                                            S.empty_dst.as<int32_t>());
    // long rows in order
    SPMM_TRY(lpos.alloc(std::max(n_long, 1) * sizeof(int32_t), s));
    k_scatter_flagged<<<g1(M), 256, 0, s>>>(fl.as<int32_t>(), pl.as<int32_t>(), nullptr, M, lpos.as<int32_t>());
    SPMM_CUDA(cudaGetLastError());
    // segments: tasks and chunk groups
    SPMM_TRY(tasks.alloc((n_long + 1) * sizeof(int32_t), s));
    SPMM_TRY(groups.alloc((n_long + 1) * sizeof(int32_t), s));
    SPMM_TRY(taskbase.alloc((n_long + 2) * sizeof(int32_t), s));
    SPMM_TRY(S.pslot_ptr.alloc((n_long + 2) * sizeof(int32_t), s));
    k_segment_counts<<<g1(n_long + 1), 256, 0, s>>>(lpos.as<int32_t>(), n_long, ps.as<int32_t>(), n_short, rowptr,
                                                    split, rpw, tasks.as<int32_t>(), groups.as<int32_t>());
    SPMM_CUDA(cudaGetLastError());
    int32_t n_tasks = 0, n_groups = 0;
    SPMM_TRY(exclusive_scan_i32(tasks.as<int32_t>(), taskbase.as<int32_t>(), n_long + 1, &n_tasks, s));
    SPMM_TRY(exclusive_scan_i32(groups.as<int32_t>(), S.pslot_ptr.as<int32_t>(), n_long + 1, &n_groups, s));
    S.n_tasks = n_tasks;
    S.n_pslots = n_groups;
    S.n_long = n_long;
    SPMM_TRY(S.units.alloc(std::max<int64_t>((int64_t)n_tasks * rpw, 1) * sizeof(int4), s));
    SPMM_TRY(S.long_dst.alloc(std::max(n_long, 1) * sizeof(int32_t), s));
    if (n_tasks > 0) {
        k_fill_int4<<<g1((int64_t)n_tasks * rpw), 256, 0, s>>>(S.units.as<int4>(), (int64_t)n_tasks * rpw,
                                                                make_int4(0, 0, NOSTORE, 0));
        k_fill_short<<<g1(M), 256, 0, s>>>(fs.as<int32_t>(), ps.as<int32_t>(), pl.as<int32_t>(), lpos.as<int32_t>(),
                                           taskbase.as<int32_t>(), rowptr, h->perm.as<int32_t>(), M, rpw,
                                           S.units.as<int4>());
        if (n_long > 0)
            k_fill_long<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div((int64_t)n_long * 32, 256), 148 * 32)),
                          256, 0, s>>>(lpos.as<int32_t>(), n_long, ps.as<int32_t>(), taskbase.as<int32_t>(),
                                       S.pslot_ptr.as<int32_t>(), rowptr, h->perm.as<int32_t>(), split, rpw,
                                       S.units.as<int4>(), S.long_dst.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    S.rpw = rpw;
    return SPMM_OK;
}

using SpmmKernel = void (*)(const int4 *, int64_t, const int2 *, const float4 *, float4 *, int32_t, float4 *,
                            unsigned int *);

template <int V, bool MASK, int SCHED, int VAR>
SpmmKernel pick_g(int G) {
    switch (G) {
        case 1: return k_spmm<V, 1, MASK, SCHED, VAR>;
        case 2: return k_spmm<V, 2, MASK, SCHED, VAR>;
        case 4: return k_spmm<V, 4, MASK, SCHED, VAR>;
        case 8: return k_spmm<V, 8, MASK, SCHED, VAR>;
        case 16: return k_spmm<V, 16, MASK, SCHED, VAR>;
        default: return k_spmm<V, 32, MASK, SCHED, VAR>;
    }
}
// run-time knobs (tuning experiments; defaults are the measured best): SPMM_SCHED (0 per-warp claiming,
// 1 CTA-contiguous queue), SPMM_VARIANT (bit 0 L2 cache hints, bit 1 U=4)
template <int V, bool MASK>
SpmmKernel pick_gs(int G, int sched, int var) {
    if (sched) return pick_g<V, MASK, 1, 0>(G);
    switch (var) {
        case 1: return pick_g<V, MASK, 0, 1>(G);
        case 2: return pick_g<V, MASK, 0, 2>(G);
        case 3: return pick_g<V, MASK, 0, 3>(G);
        default: return pick_g<V, MASK, 0, 0>(G);
    }
}

using PsKernel = void (*)(const int4 *, const int32_t *, const int32_t *, const int32_t *, int64_t, const int2 *,
                          const float4 *, float4 *, int32_t, float4 *, unsigned int *);
PsKernel pick_ps(int V, int G) {
    if (G == 8) return V == 4 ? k_spmm_ps<4, 8> : V == 3 ? k_spmm_ps<3, 8> : V == 2 ? k_spmm_ps<2, 8> : k_spmm_ps<1, 8>;
    if (G == 16) return V == 4 ? k_spmm_ps<4, 16> : V == 3 ? k_spmm_ps<3, 16> : V == 2 ? k_spmm_ps<2, 16> : k_spmm_ps<1, 16>;
    if (G == 32) return V == 4 ? k_spmm_ps<4, 32> : V == 3 ? k_spmm_ps<3, 32> : V == 2 ? k_spmm_ps<2, 32> : k_spmm_ps<1, 32>;
    return nullptr;
}

struct Config {
    SpmmKernel kern;
    int V, G, tiles;
};

// Exact fit 4*V*G == K with V in {4,3,2,1} and G a power of two <= 32, preferring G >= 8 so that one
// vector load of a group covers whole 128-byte lines (G*16 B >= 128 B: an L1 wavefront per line, measured
// to halve L1 data-pipe load at K=64); else V=4 with a masked column tail.
Config choose(int32_t K4, int sched, int var) {
    for (int V = 4; V >= 1; --V) {
        if (K4 % V) continue;
        int G = K4 / V;
        if (G >= 8 && G <= 32 && (G & (G - 1)) == 0) {
            SpmmKernel k = V == 4 ? pick_gs<4, false>(G, sched, var) : V == 3 ? pick_gs<3, false>(G, sched, var)
                         : V == 2 ? pick_gs<2, false>(G, sched, var) : pick_gs<1, false>(G, sched, var);
            return {k, V, G, 1};
        }
    }
    for (int V = 4; V >= 1; --V) {
        if (K4 % V) continue;
        int G = K4 / V;
        if (G >= 1 && G <= 32 && (G & (G - 1)) == 0) {
            SpmmKernel k = V == 4 ? pick_gs<4, false>(G, sched, var) : V == 3 ? pick_gs<3, false>(G, sched, var)
                         : V == 2 ? pick_gs<2, false>(G, sched, var) : pick_gs<1, false>(G, sched, var);
            return {k, V, G, 1};
        }
    }
    int G = 1;
    while (G < 32 && 4 * G < K4) G <<= 1;
    int tiles = (int)ceil_div(K4, 4 * G);
    return {pick_gs<4, true>(G, sched, var), 4, G, tiles};
}

}  // namespace

static spmm_status launch_ps(spmm_ctx *h, const float *B, int64_t K, float *C, cudaStream_t s, int V, int G,
                             int32_t *launches) {
    const int32_t K4 = (int32_t)(K / 4);
    static const int pr = [] { const char *e = getenv("SPMM_PANEL_ROWS"); return e ? atoi(e) : 256; }();
    static const int smem_kb = [] { const char *e = getenv("SPMM_PS_SMEM_KB"); return e ? atoi(e) : 200; }();
    const int32_t cap = (int32_t)std::max<int64_t>(1, ((int64_t)smem_kb * 1024) / (K * 4));
    if (h->psched.K != K) SPMM_TRY(build_panel_schedule(h, K, pr, cap, s));
    const PanelSchedule &S = h->psched;
    float4 *C4 = reinterpret_cast<float4 *>(C);
    float4 *P4 = nullptr;
    if (S.n_pslots > 0) {
        const size_t need = (size_t)S.n_pslots * K * sizeof(float);
        if (h->partials.bytes < need) SPMM_TRY(h->partials.alloc(need, s));
        P4 = h->partials.as<float4>();
    }
    if (S.n_empty > 0) {
        k_zero_rows<<<g1(S.n_empty * K4), 256, 0, s>>>(S.empty_dst.as<int32_t>(), S.n_empty, K4, C4);
        SPMM_CUDA(cudaGetLastError());
        ++*launches;
    }
    if (S.n_units > 0) {
        PsKernel kern = pick_ps(V, G);
        const size_t smem = (size_t)cap * K * sizeof(float);
        SPMM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        if (h->counters.bytes < sizeof(unsigned int)) SPMM_TRY(h->counters.alloc(64 * sizeof(unsigned int), s));
        SPMM_CUDA(cudaMemsetAsync(h->counters.p, 0, sizeof(unsigned int), s));
        kern<<<(unsigned)std::min<int64_t>(h->num_sms, S.n_panels), PS_THREADS, smem, s>>>(
            S.units.as<int4>(), S.panel_unit_ptr.as<int32_t>(), S.stage_ptr.as<int32_t>(), S.staged_cols.as<int32_t>(),
            S.n_panels, S.cv_ps.as<int2>(), reinterpret_cast<const float4 *>(B), C4, K4, P4,
            h->counters.as<unsigned int>());
        SPMM_CUDA(cudaGetLastError());
        ++*launches;
    }
    if (S.n_long > 0) {
        k_combine<<<(unsigned)S.n_long, 128, 0, s>>>(P4, S.pslot_ptr.as<int32_t>(), S.long_dst.as<int32_t>(), C4, K4);
        SPMM_CUDA(cudaGetLastError());
        ++*launches;
    }
    return SPMM_OK;
}

spmm_status launch_spmm(spmm_ctx *h, const float *B, int64_t K, float *C, cudaStream_t s, int32_t *launches) {
    *launches = 0;
    const int64_t M = h->M;
    if (M == 0) return SPMM_OK;
    const int32_t K4 = (int32_t)(K / 4);
    static const int sched = [] { const char *e = getenv("SPMM_SCHED"); return e ? atoi(e) : 0; }();
    static const int var = [] { const char *e = getenv("SPMM_VARIANT"); return e ? atoi(e) : 0; }();
    const Config cfg = choose(K4, sched, var);
    static const int kmode = [] { const char *e = getenv("SPMM_KERNEL"); return e ? atoi(e) : 1; }();
    if (kmode == 2 && cfg.tiles == 1 && pick_ps(cfg.V, cfg.G) != nullptr) return launch_ps(h, B, K, C, s, cfg.V, cfg.G, launches);
    const int32_t rpw = 32 / cfg.G;
    if (h->sched.rpw != rpw) SPMM_TRY(build_schedule(h, rpw, s));
    const Schedule &S = h->sched;
    float4 *C4 = reinterpret_cast<float4 *>(C);
    float4 *P4 = nullptr;
    if (S.n_pslots > 0) {
        const size_t need = (size_t)S.n_pslots * K * sizeof(float);
        if (h->partials.bytes < need) SPMM_TRY(h->partials.alloc(need, s));
        P4 = h->partials.as<float4>();
    }
    if (S.n_empty > 0) {
        k_zero_rows<<<g1(S.n_empty * K4), 256, 0, s>>>(S.empty_dst.as<int32_t>(), S.n_empty, K4, C4);
        SPMM_CUDA(cudaGetLastError());
        ++*launches;
    }
    if (S.n_tasks > 0) {
        int occ = 0;
        SPMM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, cfg.kern, SPMM_THREADS, 0));
        occ = std::max(occ, 1);
        const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(S.n_tasks, SPMM_THREADS / 32),
                                                                      (int64_t)h->num_sms * occ));
        const dim3 grid((unsigned)blocks, (unsigned)cfg.tiles);
        if (h->counters.bytes < (size_t)cfg.tiles * sizeof(unsigned int))
            SPMM_TRY(h->counters.alloc(64 * sizeof(unsigned int), s));
        SPMM_CUDA(cudaMemsetAsync(h->counters.p, 0, (size_t)cfg.tiles * sizeof(unsigned int), s));
        cfg.kern<<<grid, SPMM_THREADS, 0, s>>>(S.units.as<int4>(), S.n_tasks, h->cv_p.as<int2>(),
                                               reinterpret_cast<const float4 *>(B), C4, K4, P4,
                                               h->counters.as<unsigned int>());
        SPMM_CUDA(cudaGetLastError());
        ++*launches;
    }
    if (S.n_long > 0) {
        k_combine<<<(unsigned)S.n_long, 128, 0, s>>>(P4, S.pslot_ptr.as<int32_t>(), S.long_dst.as<int32_t>(), C4, K4);
        SPMM_CUDA(cudaGetLastError());
        ++*launches;
    }
    return SPMM_OK;
}

}  // namespace spmm
