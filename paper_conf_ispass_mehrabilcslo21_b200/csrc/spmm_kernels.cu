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
#include <cmath>
#include <climits>
#include <cstdlib>
#include <vector>

namespace spmm {
namespace {

constexpr int SPMM_THREADS = 256;
constexpr int32_t NOSTORE = INT_MIN;
constexpr int SORT_WIN = 32;          // a7: short rows sorted by length within windows of this many positions

// ---- per-lane vectors: W = 4 floats (LDG.128) or W = 8 floats (sm_100 LDG.E.ENL2.256) ---------------
struct float8 {
    float4 lo, hi;
};
template <int W> struct VecT;
template <> struct VecT<4> { using T = float4; };
template <> struct VecT<8> { using T = float8; };

__device__ __forceinline__ void fma4(float a, const float4 &b, float4 &acc) {
    float2 lo = __ffma2_rn(make_float2(a, a), make_float2(b.x, b.y), make_float2(acc.x, acc.y));
    float2 hi = __ffma2_rn(make_float2(a, a), make_float2(b.z, b.w), make_float2(acc.z, acc.w));
    acc.x = lo.x; acc.y = lo.y; acc.z = hi.x; acc.w = hi.y;
}
__device__ __forceinline__ void vfma(float a, const float4 &b, float4 &acc) { fma4(a, b, acc); }
__device__ __forceinline__ void vfma(float a, const float8 &b, float8 &acc) {
    fma4(a, b.lo, acc.lo);
    fma4(a, b.hi, acc.hi);
}
__device__ __forceinline__ void vzero(float4 &a) { a = make_float4(0.f, 0.f, 0.f, 0.f); }
__device__ __forceinline__ void vzero(float8 &a) { vzero(a.lo); vzero(a.hi); }
__device__ __forceinline__ void xadd(float4 &a, int off) {
    a.x += __shfl_xor_sync(0xffffffffu, a.x, off);
    a.y += __shfl_xor_sync(0xffffffffu, a.y, off);
    a.z += __shfl_xor_sync(0xffffffffu, a.z, off);
    a.w += __shfl_xor_sync(0xffffffffu, a.w, off);
}
__device__ __forceinline__ void xadd(float8 &a, int off) { xadd(a.lo, off); xadd(a.hi, off); }
__device__ __forceinline__ void vstore_cs(float4 *p, const float4 &v) { __stcs(p, v); }
__device__ __forceinline__ void vstore_cs(float8 *p, const float8 &v) {
    asm volatile("st.global.cs.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(v.lo.x), "f"(v.lo.y),
                 "f"(v.lo.z), "f"(v.lo.w), "f"(v.hi.x), "f"(v.hi.y), "f"(v.hi.z), "f"(v.hi.w) : "memory");
}
__device__ __forceinline__ void vstore(float4 *p, const float4 &v) { *p = v; }
// NVLS multicast store (SURVEY §8(f) f2 ii): p is a multicast address -- one store reaches the buffer on every
// member GPU through the NVSwitch (multimem.st, at most 128 bits per instruction)
__device__ __forceinline__ void mcstore(float4 *p, const float4 &v) {
    asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
                 "f"(v.w) : "memory");
}
__device__ __forceinline__ void mcstore(float8 *p, const float8 &v) {
    mcstore(reinterpret_cast<float4 *>(p), v.lo);
    mcstore(reinterpret_cast<float4 *>(p) + 1, v.hi);
}
// a store to extra destination i of spmm_run_to (mc bit i: a multicast address)
template <class VT>
__device__ __forceinline__ void xstore(VT *p, const VT &v, bool mc) {
    if (mc) mcstore(p, v);
    else vstore_cs(p, v);
}
__device__ __forceinline__ void vstore(float8 *p, const float8 &v) {
    asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(v.lo.x), "f"(v.lo.y),
                 "f"(v.lo.z), "f"(v.lo.w), "f"(v.hi.x), "f"(v.hi.y), "f"(v.hi.z), "f"(v.hi.w) : "memory");
}

// Loads of the inner loop: read-only (ld.global.nc) B vectors -- W = 8: one 256-bit load per lane (sm_100
// LDG.E.ENL2.256, which tools/ldpathprobe.cu measures at twice the bytes per SM clock of 128-bit loads for the same
// gather), W = 4: LDG.128 -- and 8-byte (col, val) pairs.
__device__ __forceinline__ float4 ld_b(const float4 *ptr) { return __ldg(ptr); }
__device__ __forceinline__ float8 ld_b(const float8 *ptr) {
    float8 r;
    asm("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=f"(r.lo.x), "=f"(r.lo.y), "=f"(r.lo.z), "=f"(r.lo.w), "=f"(r.hi.x), "=f"(r.hi.y), "=f"(r.hi.z), "=f"(r.hi.w)
        : "l"(ptr));
    return r;
}
__device__ __forceinline__ int2 ld_cv(const int2 *ptr) { return __ldg(ptr); }

// B row offset in W-float vectors (64-bit: B exceeds 4 GB at C5).  V = 1: unsigned 32 x 32 -> 64-bit (IMAD.WIDE.U32,
// no sign extensions; column ids and strides are non-negative); V >= 2: signed (the unsigned form makes ptxas spill
// in the K = 128 fused kernel)
template <int V>
__device__ __forceinline__ size_t brow(int32_t col, int32_t KV) {
    if constexpr (V == 1) return (size_t)(uint32_t)col * (uint32_t)KV;
    else return (size_t)col * KV;
}

// One work unit per lane group: the G lanes of group g own the unit u = (start, len, dst) and the V vectors
// (VT = W floats each) col0 + v*G of its C row (colok: inside K; indices in VT units, KV = K / W per row).
// Per nnz the group broadcasts the (col, val) pair with two shuffles from a register batch prefetched one
// batch ahead (coalesced 8-byte loads of the interleaved permuted CSR), issues V coalesced W*4-byte loads of
// the B row (G*W*4 contiguous bytes per group and vector: whole 128-byte lines), then W*V/2 packed FFMA2
// -- each accumulator is a sequential chain in ascending j, the order of the oracle's definition
// (oracle.c c1).  U nnz per inner step: U*V independent B loads are issued before the first FMA.  The trip
// count is warp-uniform (groups past their own length are predicated off), so the shuffles stay warp-wide.
// Store: a whole row -> C[perm[p]] (streaming store); a chunk group of a long row -> the warp's groups
// are reduced by a fixed xor butterfly and group 0 writes the partial.
template <int V, int G, int U, class VT, bool MD = false>
__device__ __forceinline__ void spmm_unit(const int4 u, const int g, const int gl, const int col0, const bool (&colok)[V],
                                          const int2 *__restrict__ cv, const VT *__restrict__ BV,
                                          VT *__restrict__ CV, const int32_t KV, const int32_t LC,
                                          VT *__restrict__ PV, const CExtra &cx) {
    constexpr int BATCH = (G >= 8 ? G : 8) >= U ? (G >= 8 ? G : 8) : U;   // (col, val) pairs per group per batch
    constexpr int PL = BATCH / G;                // pairs held per lane
    const int32_t start = u.x, len = u.y, dst = u.z;
    const int32_t maxlen = (int32_t)__reduce_max_sync(0xffffffffu, (unsigned)len);
    VT acc[V];
#pragma unroll
    for (int v = 0; v < V; ++v) vzero(acc[v]);
    int2 cur[PL];
#pragma unroll
    for (int p = 0; p < PL; ++p) {
        const int32_t o = p * G + gl;
        cur[p] = o < len ? ld_cv(cv + start + o) : make_int2(0, 0);
    }
    for (int32_t b0 = 0; b0 < maxlen; b0 += BATCH) {
        int2 nxt[PL];
#pragma unroll
        for (int p = 0; p < PL; ++p) {
            const int32_t o = b0 + BATCH + p * G + gl;
            nxt[p] = o < len ? ld_cv(cv + start + o) : make_int2(0, 0);
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
                VT x[U][V];
#pragma unroll
                for (int w = 0; w < U; ++w) {
                    const VT *b = BV + brow<V>(col[w], KV) + col0;
#pragma unroll
                    for (int v = 0; v < V; ++v) {
                        if (colok[v]) x[w][v] = ld_b(b + v * G);
                        else vzero(x[w][v]);
                    }
                }
#pragma unroll
                for (int w = 0; w < U; ++w)
#pragma unroll
                    for (int v = 0; v < V; ++v) vfma(a[w], x[w][v], acc[v]);
            } else if (rem > 0) {                    // the group's tail
#pragma unroll
                for (int w = 0; w < U - 1; ++w) {
                    if (w < rem) {
                        const VT *b = BV + brow<V>(col[w], KV) + col0;
#pragma unroll
                        for (int v = 0; v < V; ++v)
                            if (colok[v]) vfma(a[w], ld_b(b + v * G), acc[v]);
                    }
                }
            }
        }
#pragma unroll
        for (int p = 0; p < PL; ++p) cur[p] = nxt[p];
    }
    if (dst >= 0) {                                    // a whole row: C[perm[p]] (+ the extra destinations)
        if (!MD || !cx.skip_main) {
#pragma unroll
            for (int v = 0; v < V; ++v)
                if (colok[v]) vstore_cs(CV + (size_t)dst * LC + col0 + v * G, acc[v]);
        }
        if constexpr (MD) {   // spmm_run_to instantiations only: no cost for plain runs
#pragma unroll
            for (int i = 0; i < SPMM_MAX_CDST - 1; ++i) {   // constant indices: cx stays in parameter space
                if (i >= cx.n) break;
                VT *X = reinterpret_cast<VT *>(cx.p[i]);
                const bool mc = (cx.mc >> i) & 1u;
#pragma unroll
                for (int v = 0; v < V; ++v)
                    if (colok[v]) xstore(X + (size_t)dst * LC + col0 + v * G, acc[v], mc);
            }
        }
    } else if (dst != NOSTORE) {                       // chunk group of a long row (warp-uniform)
#pragma unroll
        for (int off = G; off < 32; off <<= 1) {       // fixed butterfly: ((c0+c1)+(c2+c3))...
#pragma unroll
            for (int v = 0; v < V; ++v) xadd(acc[v], off);
        }
        if (g == 0) {
            const int64_t slot = -(int64_t)dst - 1;
#pragma unroll
            for (int v = 0; v < V; ++v)
                if (colok[v]) vstore(PV + slot * KV + col0 + v * G, acc[v]);
        }
    }
}

// A fused unit (row fusion, Schedule): the G lanes of group g walk the sorted union of the columns of R
// consecutive rows once.  Per union record the group broadcasts (col, mask, v_0..v_{R-1}) with R + 2
// shuffles, loads the B row once (V vectors per lane) and feeds member r's accumulator with v_r where mask
// bit r is set (predicated FFMA2: a member without the column adds nothing, so each member's accumulator is
// the same sequential ascending-column chain as in spmm_unit -- bit-identical C).  Stores: C[gdst[r]].
template <int R> struct RecT;
template <> struct RecT<2> { int4 a; };
template <> struct RecT<4> { int4 a, b; };
__device__ __forceinline__ RecT<2> ld_rec(const RecT<2> *p) { return RecT<2>{__ldg(&p->a)}; }
__device__ __forceinline__ RecT<4> ld_rec(const RecT<4> *p) { return RecT<4>{__ldg(&p->a), __ldg(&p->b)}; }
__device__ __forceinline__ int rec_word(const RecT<2> &r, int i) {
    return i == 0 ? r.a.x : i == 1 ? r.a.y : i == 2 ? r.a.z : r.a.w;
}
__device__ __forceinline__ int rec_word(const RecT<4> &r, int i) {
    return i == 0 ? r.a.x : i == 1 ? r.a.y : i == 2 ? r.a.z : i == 3 ? r.a.w : i == 4 ? r.b.x : r.b.y;
}
__device__ __forceinline__ RecT<2> rec_zero(RecT<2>) { return RecT<2>{make_int4(0, 0, 0, 0)}; }
__device__ __forceinline__ RecT<4> rec_zero(RecT<4>) { return RecT<4>{make_int4(0, 0, 0, 0), make_int4(0, 0, 0, 0)}; }

template <int V, int G, int R, int U, class VT, bool MD = false>
__device__ __forceinline__ void spmm_unit_fused(const int4 u, const int g, const int gl, const int col0,
                                                const bool (&colok)[V], const RecT<R> *__restrict__ recs,
                                                const int32_t *__restrict__ gdst, const VT *__restrict__ BV,
                                                VT *__restrict__ CV, const int32_t KV, const int32_t LC,
                                                const CExtra &cx) {
    constexpr int BATCH = G >= 8 ? G : 8;        // records per group per batch
    constexpr int PL = BATCH / G;                // records held per lane
    const int32_t start = u.x, len = u.y, gid = u.z;
    const int32_t maxlen = (int32_t)__reduce_max_sync(0xffffffffu, (unsigned)len);
    VT acc[R][V];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
        for (int v = 0; v < V; ++v) vzero(acc[r][v]);
    RecT<R> cur[PL];
#pragma unroll
    for (int p = 0; p < PL; ++p) {
        const int32_t o = p * G + gl;
        cur[p] = o < len ? ld_rec(recs + start + o) : rec_zero(RecT<R>{});
    }
    for (int32_t b0 = 0; b0 < maxlen; b0 += BATCH) {
        RecT<R> nxt[PL];
#pragma unroll
        for (int p = 0; p < PL; ++p) {
            const int32_t o = b0 + BATCH + p * G + gl;
            nxt[p] = o < len ? ld_rec(recs + start + o) : rec_zero(RecT<R>{});
        }
#pragma unroll
        for (int q0 = 0; q0 < BATCH; q0 += U) {
            int32_t col[U];
            uint32_t mask[U];
            float a[U][R];
#pragma unroll
            for (int w = 0; w < U; ++w) {
                const int qq = q0 + w;
                const int src = g * G + (qq % G);
                col[w] = __shfl_sync(0xffffffffu, rec_word(cur[qq / G], 0), src);
                mask[w] = (uint32_t)__shfl_sync(0xffffffffu, rec_word(cur[qq / G], 1), src);
#pragma unroll
                for (int r = 0; r < R; ++r)
                    a[w][r] = __int_as_float(__shfl_sync(0xffffffffu, rec_word(cur[qq / G], 2 + r), src));
            }
            const int32_t rem = len - (b0 + q0);
            if (rem > 0) {
                VT x[U][V];
#pragma unroll
                for (int w = 0; w < U; ++w) {
                    const VT *b = BV + brow<V>(col[w], KV) + col0;
#pragma unroll
                    for (int v = 0; v < V; ++v) {
                        if (colok[v] && w < rem) x[w][v] = ld_b(b + v * G);
                        else if (V > 1) vzero(x[w][v]);   // V = 1: unused (the FFMA2s below are predicated by
                                                          // the same w < rem); V = 2: keeps ptxas from spilling
                    }
                }

#pragma unroll
                for (int w = 0; w < U; ++w)
#pragma unroll
                    for (int r = 0; r < R; ++r)
                        if (w < rem && ((mask[w] >> r) & 1u))
#pragma unroll
                            for (int v = 0; v < V; ++v) vfma(a[w][r], x[w][v], acc[r][v]);
            }
        }
#pragma unroll
        for (int p = 0; p < PL; ++p) cur[p] = nxt[p];
    }
    if (gid >= 0) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const int32_t dst = __ldg(gdst + (size_t)gid * R + r);
            if (dst >= 0) {
                if (!MD || !cx.skip_main) {
#pragma unroll
                    for (int v = 0; v < V; ++v)
                        if (colok[v]) vstore_cs(CV + (size_t)dst * LC + col0 + v * G, acc[r][v]);
                }
                if constexpr (MD) {   // spmm_run_to instantiations only: no cost for plain runs
#pragma unroll
                    for (int i = 0; i < SPMM_MAX_CDST - 1; ++i) {   // constant indices: cx stays in param space
                        if (i >= cx.n) break;
                        VT *X = reinterpret_cast<VT *>(cx.p[i]);
                        const bool mc = (cx.mc >> i) & 1u;
#pragma unroll
                        for (int v = 0; v < V; ++v)
                            if (colok[v]) xstore(X + (size_t)dst * LC + col0 + v * G, acc[r][v], mc);
                    }
                }
            }
        }
    }
}

// The row-group SpMM over the a7 warp-task list.  V vectors of W floats per lane, G lanes per unit, MASK: column
// tail present (K not a multiple of W*V*G, several column tiles).  Warp tasks are claimed dynamically (one atomicAdd
// per task on a per-column-tile counter), so the set of tasks in flight stays a narrow window of the permuted
// order whatever the task costs: the order's B-row locality survives into L2 and no warp is left with a long
// static tail.
// FR > 1: the kernel also runs fused tasks (row fusion, Schedule) -- a task's type is its first unit's w field
// (1 = fused), uniform over the warp by construction.  The fused kernel needs > 80 registers (2 CTAs/SM), so it
// takes a two-deep task pipeline with an L2 prefetch (prefetch.global.L2) of the next task's record range issued
// one task ahead (measured 0.336 -> 0.321 ms at C2, K = 64; the unfused kernel at 3 CTAs/SM gains nothing from it).
// MD: spmm_run_to instantiations (extra C destinations), so plain runs carry no extra code.
template <int V, int G, bool MASK, int W, int FR, bool MD>
__global__ void __launch_bounds__(SPMM_THREADS, FR > 1 ? 2 : 3) k_spmm(const int4 *__restrict__ units, int64_t n_tasks,
                                                       const int2 *__restrict__ cv, const float4 *__restrict__ B4,
                                                       float4 *__restrict__ C4, int32_t K4, int32_t ldc4,
                                                       float4 *__restrict__ P4, unsigned int *__restrict__ counter,
                                                       const int4 *__restrict__ recs,
                                                       const int32_t *__restrict__ gdst, const CExtra cx) {
    using VT = typename VecT<W>::T;
    constexpr int RPW = 32 / G;
    constexpr int CTV = V * G;
    constexpr int U = V * W >= 12 ? 2 : 4;        // nnz per inner step (B loads in flight per lane: U*V)
    constexpr int FU = V == 1 ? 4 : 2;            // union records per inner step of a fused unit
    constexpr bool PF = FR > 1;
    const int32_t KV = K4 * 4 / W, LC = ldc4 * 4 / W;   // B row / C row strides in W-float vectors
    const int lane = threadIdx.x & 31;
    const int g = lane / G, gl = lane % G;
    const int col0 = blockIdx.y * CTV + gl;      // this lane's first vector column; then + v*G
    bool colok[V];
#pragma unroll
    for (int v = 0; v < V; ++v) colok[v] = !MASK || (col0 + v * G < KV);

    unsigned int tk = 0;
    if (lane == 0) tk = atomicAdd(counter + blockIdx.y, 1u);
    tk = __shfl_sync(0xffffffffu, tk, 0);
    int64_t t = tk;
    int4 u = t < n_tasks ? __ldg(units + t * RPW + g) : make_int4(0, 0, NOSTORE, 0);
    int64_t t1 = 0;
    int4 u1 = make_int4(0, 0, NOSTORE, 0);
    if (PF) {
        if (lane == 0) tk = atomicAdd(counter + blockIdx.y, 1u);
        t1 = __shfl_sync(0xffffffffu, tk, 0);
        u1 = t1 < n_tasks ? __ldg(units + t1 * RPW + g) : make_int4(0, 0, NOSTORE, 0);
    }
    while (t < n_tasks) {
        // claim and fetch the next task first, so its latency hides behind this one
        int64_t t_next;
        int4 u_next;
        if (PF) {
            // two-deep: u1 (fetched one task ago) is in registers -- prefetch its A range into L2, then
            // claim the task after it
            if (t1 < n_tasks && u1.y > 0) {
                const bool f1 = FR > 1 && u1.w == 1;
                const int rb = f1 ? 16 * (FR / 2) : 8;
                const char *lo = f1 ? reinterpret_cast<const char *>(recs) + (size_t)u1.x * rb
                                    : reinterpret_cast<const char *>(cv) + (size_t)u1.x * 8;
                const size_t l0 = reinterpret_cast<uintptr_t>(lo) >> 7;
                const size_t l1 = (reinterpret_cast<uintptr_t>(lo) + (size_t)u1.y * rb - 1) >> 7;
                for (size_t l = l0 + gl; l <= l1; l += G)
                    asm volatile("prefetch.global.L2 [%0];" ::"l"(reinterpret_cast<const void *>(l << 7)));
            }
            if (lane == 0) tk = atomicAdd(counter + blockIdx.y, 1u);
            const int64_t t2 = __shfl_sync(0xffffffffu, tk, 0);
            const int4 u2 = t2 < n_tasks ? __ldg(units + t2 * RPW + g) : make_int4(0, 0, NOSTORE, 0);
            t_next = t1;
            u_next = u1;
            t1 = t2;
            u1 = u2;
        } else {
            if (lane == 0) tk = atomicAdd(counter + blockIdx.y, 1u);
            t_next = __shfl_sync(0xffffffffu, tk, 0);
            u_next = t_next < n_tasks ? __ldg(units + t_next * RPW + g) : make_int4(0, 0, NOSTORE, 0);
        }
        bool fused = false;
        if (FR > 1) fused = __shfl_sync(0xffffffffu, u.w, 0) == 1;
        if (FR > 1 && fused) {
            spmm_unit_fused<V, G, (FR > 1 ? FR : 2), FU, VT, MD>(u, g, gl, col0, colok,
                                                     reinterpret_cast<const RecT<(FR > 1 ? FR : 2)> *>(recs), gdst,
                                                     reinterpret_cast<const VT *>(B4), reinterpret_cast<VT *>(C4), KV,
                                                     LC, cx);
        } else {
            spmm_unit<V, G, U, VT, MD>(u, g, gl, col0, colok, cv, reinterpret_cast<const VT *>(B4),
                                       reinterpret_cast<VT *>(C4), KV, LC, reinterpret_cast<VT *>(P4), cx);
        }
        t = t_next;
        u = u_next;
    }
}

// Pairwise (binary-counter) combine of a long row's chunk-group partials, fixed order -> deterministic;
// rounding grows with log2(#groups).  One warp per long row (8 rows per CTA), lane per float4
// column of C.
__global__ void __launch_bounds__(256) k_combine(const float4 *__restrict__ P4, const int32_t *__restrict__ pslot_ptr,
                                                 const int32_t *__restrict__ long_dst, int64_t n_long,
                                                 float4 *__restrict__ C4, int32_t K4, int32_t ldc4, const CExtra cx) {
    const int lane = threadIdx.x & 31;
    for (int64_t l = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; l < n_long;
         l += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int32_t c0 = pslot_ptr[l], c1 = pslot_ptr[l + 1];
        float4 *dst = C4 + (size_t)long_dst[l] * ldc4;
        for (int32_t col = lane; col < K4; col += 32) {
            float4 stk[24];
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
            if (!cx.skip_main) __stcs(dst + col, r);
#pragma unroll
            for (int i = 0; i < SPMM_MAX_CDST - 1; ++i)
                if (i < cx.n) xstore(cx.p[i] + (size_t)long_dst[l] * ldc4 + col, r, (cx.mc >> i) & 1u);
        }
    }
}

// Empty rows: zero-fill their C rows.  Warp per row: each lane loads one of 32 consecutive row ids (one coalesced
// load per 32 rows), then the warp walks them, storing each row's K/4 float4 with consecutive lanes (coalesced
// streaming stores).  (Round 1 strided the grid over flattened (row, column) pairs, so every store of a thread needed
// a fresh L2 load of its row id: ≈ 0.8 TB/s, 6 ms for C5's 3.9 GB of empty C rows -- the floor of a step whose
// SpMM is short, e.g. the last shard of C5 at 8 GPUs.)
__global__ void k_zero_rows(const int32_t *__restrict__ rows, int64_t n, int32_t K4, int32_t ldc4,
                            float4 *__restrict__ C4, const CExtra cx) {
    const int lane = threadIdx.x & 31;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int64_t base = warp * 32; base < n; base += nwarps * 32) {
        const int32_t mine = base + lane < n ? __ldg(rows + base + lane) : 0;
        const int cnt = n - base < 32 ? (int)(n - base) : 32;
        for (int j = 0; j < cnt; ++j) {
            const size_t o = (size_t)__shfl_sync(0xffffffffu, mine, j) * ldc4;
            for (int32_t c = lane; c < K4; c += 32) {
                if (!cx.skip_main) __stcs(C4 + o + c, z);
#pragma unroll
                for (int e = 0; e < SPMM_MAX_CDST - 1; ++e)
                    if (e < cx.n) xstore(cx.p[e] + o + c, z, (cx.mc >> e) & 1u);
            }
        }
    }
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

// lengths of the short rows in compacted (position) order
__global__ void k_short_len(const int32_t *is_short, const int32_t *sp, const int32_t *rowptr, int64_t M, int32_t *slen) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x)
        if (is_short[p]) slen[sp[p]] = rowptr[p + 1] - rowptr[p];
}

// Short rows -> units.  The run of short rows of a segment is cut into windows of `win` consecutive rows
// (win a multiple of RPW; 0 = no windows); inside a window the rows are placed by descending length (ties:
// position), so the RPW rows of a warp task have similar lengths and the warp-uniform trip count (the
// longest unit) wastes few lane slots -- the paper's load-balance concern applied within a
// window of `win` rows, which keeps the permuted order's locality (all rows of a window run at about the
// same time).  The per-row arithmetic is unchanged (one unit per row).
__global__ void k_fill_short(const int32_t *is_short, const int32_t *sp, const int32_t *lidx, const int32_t *lpos,
                             const int32_t *taskbase, const int32_t *rowptr, const int32_t *perm, const int32_t *slen,
                             int32_t n_short, int64_t n_long, int64_t M, int32_t rpw, int32_t win, int4 *units) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        if (!is_short[p]) continue;
        const int32_t k = lidx[p];                         // long rows before p = this run's segment
        const int32_t before = k > 0 ? sp[lpos[k - 1]] : 0;
        int32_t idx = sp[p] - before;
        const int32_t len = rowptr[p + 1] - rowptr[p];
        if (win > 0) {
            const int32_t w0 = before + (idx / win) * win;
            const int32_t upto = k < n_long ? sp[lpos[k]] : n_short;   // end of this run
            const int32_t w1 = w0 + win < upto ? w0 + win : upto;
            int32_t rank = 0;
            const int32_t me = sp[p];
            for (int32_t j = w0; j < w1; ++j) {
                const int32_t lj = slen[j];
                rank += (lj > len) || (lj == len && j < me);
            }
            idx = (idx / win) * win + rank;
        }
        const int64_t task = (int64_t)taskbase[k] + idx / rpw;
        units[task * rpw + idx % rpw] = make_int4(rowptr[p], len, perm[p], 0);
    }
}

// Warp per long row: its chunk groups follow the run of short rows of its segment.  The row is cut into
// nch' = RPW * ceil(ceil(len / split) / RPW) chunks of balanced sizes (floor or ceil of len / nch', each
// <= split), so the RPW chunks of every chunk group have equal trip counts.  The cut depends only on the
// row length (and RPW), not on the row's position: C stays bit-identical under every permutation.
__global__ void k_fill_long(const int32_t *lpos, int64_t n_long, const int32_t *sp, const int32_t *taskbase,
                            const int32_t *pslot_ptr, const int32_t *rowptr, const int32_t *perm, int32_t rpw,
                            int32_t fr, int4 *units, int32_t *long_dst) {
    const int lane = threadIdx.x & 31;
    for (int64_t k = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < n_long;
         k += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int32_t p = lpos[k];
        const int32_t s_k = sp[p] - (k > 0 ? sp[lpos[k - 1]] : 0);
        const int32_t su = (s_k + fr - 1) / fr;          // short units before it (rows, or fusion groups)
        const int64_t t0 = (int64_t)taskbase[k] + (su + rpw - 1) / rpw;
        const int32_t a = rowptr[p], len = rowptr[p + 1] - a;
        const int32_t ng = pslot_ptr[k + 1] - pslot_ptr[k];
        const int32_t nch = ng * rpw, base = len / nch, extra = len % nch;
        for (int32_t c = lane; c < nch; c += 32) {
            const int32_t dst = -(pslot_ptr[k] + c / rpw) - 1;
            units[(t0 + c / rpw) * rpw + c % rpw] = make_int4(a + c * base + min(c, extra), base + (c < extra), dst, 0);
        }
        if (lane == 0) long_dst[k] = perm[p];
    }
}

__global__ void k_fill_int4(int4 *a, int64_t n, int4 v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) a[i] = v;
}

// ---- row fusion (Schedule) ------------------------------------------------------------------------
// per segment k: fusion groups ng_k = ceil(s_k / R) of its short-row run; tasks = ceil(ng_k / RPW) + chunk groups
__global__ void k_segment_counts_fused(const int32_t *lpos, int64_t n_long, const int32_t *sp, int32_t n_short,
                                       const int32_t *rowptr, int32_t split, int32_t rpw, int32_t R, int32_t *tasks,
                                       int32_t *groups, int32_t *ngroups) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k <= n_long; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t before = k > 0 ? sp[lpos[k - 1]] : 0;
        const int32_t upto = k < n_long ? sp[lpos[k]] : n_short;
        const int32_t ng = (upto - before + R - 1) / R;
        int32_t nch = 0;
        if (k < n_long) {
            const int32_t len = rowptr[lpos[k] + 1] - rowptr[lpos[k]];
            nch = (len + split - 1) / split;
        }
        const int32_t gk = (nch + rpw - 1) / rpw;
        tasks[k] = (ng + rpw - 1) / rpw + gk;
        groups[k] = gk;
        ngroups[k] = ng;
    }
}

// member slots of the fusion groups: gpos[g * R + r] = position of member r (-1: none), gseg[g] = segment
__global__ void k_group_members(const int32_t *is_short, const int32_t *sp, const int32_t *lidx, const int32_t *lpos,
                                const int32_t *gbase, int64_t M, int32_t R, int32_t *gpos, int32_t *gseg) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        if (!is_short[p]) continue;
        const int32_t k = lidx[p];
        const int32_t idx = sp[p] - (k > 0 ? sp[lpos[k - 1]] : 0);
        const int64_t g = (int64_t)gbase[k] + idx / R;
        gpos[g * R + idx % R] = (int32_t)p;
        if (idx % R == 0) gseg[g] = k;
    }
}

// R-way merge of the members' sorted column lists (strictly increasing within a row, A15).  FILL = false:
// ucnt[g] = union length, gnnz[g] = sum of member lengths; FILL = true: write the records at rbase[g] and
// the members' C rows (perm) to gdst.
template <bool FILL>
__global__ void k_union(const int32_t *gpos, int64_t n_groups, int32_t R, const int32_t *rowptr, const int2 *cv,
                        const int32_t *perm, int32_t *ucnt, int32_t *gnnz, const int32_t *rbase, int4 *recs,
                        int32_t *gdst) {
    for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < n_groups; g += (int64_t)gridDim.x * blockDim.x) {
        int32_t j[4], e[4], c[4];
        int32_t tot = 0;
        for (int r = 0; r < 4; ++r) {
            const int32_t p = r < R ? gpos[g * R + r] : -1;
            j[r] = p >= 0 ? rowptr[p] : 0;
            e[r] = p >= 0 ? rowptr[p + 1] : 0;
            c[r] = j[r] < e[r] ? cv[j[r]].x : INT_MAX;
            tot += e[r] - j[r];
            if (FILL && r < R) gdst[g * R + r] = p >= 0 ? perm[p] : NOSTORE;
        }
        int32_t n = 0;
        int4 *out = FILL ? recs + (int64_t)rbase[g] * (R / 2) : nullptr;
        for (;;) {
            const int32_t m = min(min(c[0], c[1]), min(c[2], c[3]));
            if (m == INT_MAX) break;
            int32_t mask = 0, v[4] = {0, 0, 0, 0};
            for (int r = 0; r < 4; ++r) {
                if (c[r] == m) {
                    mask |= 1 << r;
                    v[r] = cv[j[r]].y;
                    ++j[r];
                    c[r] = j[r] < e[r] ? cv[j[r]].x : INT_MAX;
                }
            }
            if (FILL) {
                if (R == 2) {
                    out[n] = make_int4(m, mask, v[0], v[1]);
                } else {
                    out[2 * n] = make_int4(m, mask, v[0], v[1]);
                    out[2 * n + 1] = make_int4(v[2], v[3], 0, 0);
                }
            }
            ++n;
        }
        if (!FILL) {
            ucnt[g] = n;
            gnnz[g] = tot;
        }
    }
}

// Fusion groups -> fused units.  As for rows (k_fill_short): the groups of a segment are cut into windows of
// `win` consecutive groups, inside which they are placed by descending union length (ties: group id).
__global__ void k_fill_fused(const int32_t *gseg, int64_t n_groups, const int32_t *gbase, const int32_t *ngroups,
                             const int32_t *taskbase, const int32_t *ucnt, const int32_t *rbase, int32_t rpw,
                             int32_t win, int4 *units) {
    for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < n_groups; g += (int64_t)gridDim.x * blockDim.x) {
        const int32_t k = gseg[g];
        const int32_t g0 = gbase[k];
        int32_t idx = (int32_t)(g - g0);
        const int32_t len = ucnt[g];
        if (win > 0) {
            const int32_t w0 = g0 + (idx / win) * win;
            const int32_t w1 = min(w0 + win, g0 + ngroups[k]);
            int32_t rank = 0;
            for (int32_t q = w0; q < w1; ++q) {
                const int32_t lq = ucnt[q];
                rank += (lq > len) || (lq == len && q < g);
            }
            idx = (idx / win) * win + rank;
        }
        const int64_t task = (int64_t)taskbase[k] + idx / rpw;
        units[task * rpw + idx % rpw] = make_int4(rbase[g], len, (int32_t)g, 1);
    }
}

inline unsigned g1(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 32)); }

// R > 1: row fusion requested (fuse_rows 0 = auto: keep it only when the unions hold <= 3/4 of the fused
// rows' nnz; 2 = always).  Falls back to R = 1 (plain row units) otherwise.
spmm_status build_schedule(spmm_ctx *h, Schedule &S, int32_t rpw, int32_t R, cudaStream_t s) {
    S.rpw = 0;
    S.fuse_req = R;
    S.fuse = 1;
    S.n_groups = S.n_records = S.fused_nnz = 0;
    S.recs.release();
    S.gdst.release();
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
    // short rows are sorted by length inside windows of 32 positions (measured: no window costs 5 % on C3 identity,
    // 32..1024 are within run-to-run noise for the locality orders -- profiles/HISTORY.md r1e)
    const int32_t win = (int32_t)ceil_div(SORT_WIN, rpw) * rpw;
    // row fusion: groups of R consecutive short rows of each run, their column unions
    DevBuf ngroups, gbase, gpos, gseg, ucnt, gnnz, rbase;
    int32_t n_fgroups = 0;
    if (R > 1 && n_short > 0) {
        SPMM_TRY(ngroups.alloc((n_long + 1) * sizeof(int32_t), s));
        SPMM_TRY(gbase.alloc((n_long + 2) * sizeof(int32_t), s));
        k_segment_counts_fused<<<g1(n_long + 1), 256, 0, s>>>(lpos.as<int32_t>(), n_long, ps.as<int32_t>(), n_short,
                                                              rowptr, split, rpw, R, tasks.as<int32_t>(),
                                                              groups.as<int32_t>(), ngroups.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(exclusive_scan_i32(ngroups.as<int32_t>(), gbase.as<int32_t>(), n_long + 1, &n_fgroups, s));
        SPMM_TRY(gpos.alloc((size_t)n_fgroups * R * sizeof(int32_t), s));
        SPMM_TRY(gseg.alloc((size_t)n_fgroups * sizeof(int32_t), s));
        SPMM_TRY(ucnt.alloc((size_t)(n_fgroups + 1) * sizeof(int32_t), s));
        SPMM_TRY(gnnz.alloc((size_t)(n_fgroups + 1) * sizeof(int32_t), s));
        SPMM_TRY(rbase.alloc((size_t)(n_fgroups + 1) * sizeof(int32_t), s));
        SPMM_CUDA(cudaMemsetAsync(gpos.p, 0xff, (size_t)n_fgroups * R * sizeof(int32_t), s));
        k_group_members<<<g1(M), 256, 0, s>>>(fs.as<int32_t>(), ps.as<int32_t>(), pl.as<int32_t>(), lpos.as<int32_t>(),
                                              gbase.as<int32_t>(), M, R, gpos.as<int32_t>(), gseg.as<int32_t>());
        k_union<false><<<g1(n_fgroups), 256, 0, s>>>(gpos.as<int32_t>(), n_fgroups, R, rowptr, h->cv_p.as<int2>(),
                                                      nullptr, ucnt.as<int32_t>(), gnnz.as<int32_t>(), nullptr,
                                                      nullptr, nullptr);
        SPMM_CUDA(cudaGetLastError());
        int32_t n_rec = 0, n_fnnz = 0;
        SPMM_TRY(exclusive_scan_i32(gnnz.as<int32_t>(), rbase.as<int32_t>(), n_fgroups, &n_fnnz, s));
        SPMM_TRY(exclusive_scan_i32(ucnt.as<int32_t>(), rbase.as<int32_t>(), n_fgroups, &n_rec, s));
        // auto: keep fusion when the unions save enough B-row loads to pay for the wider records and the
        // predicated FMAs (measured break-even: union / nnz ~0.6 at R = 4, ~0.75 at R = 2)
        const int64_t num = 3, den = R == 4 ? 5 : 4;
        const bool keep = h->params.fuse_rows == 2 || (int64_t)n_rec * den <= (int64_t)n_fnnz * num;
        if (keep) {
            S.fuse = R;
            S.n_groups = n_fgroups;
            S.n_records = n_rec;
            S.fused_nnz = n_fnnz;
            SPMM_TRY(S.recs.alloc(std::max<int64_t>((int64_t)n_rec * (R / 2), 1) * sizeof(int4), s));
            SPMM_TRY(S.gdst.alloc(std::max<int64_t>((int64_t)n_fgroups * R, 1) * sizeof(int32_t), s));
            k_union<true><<<g1(n_fgroups), 256, 0, s>>>(gpos.as<int32_t>(), n_fgroups, R, rowptr, h->cv_p.as<int2>(),
                                                         h->perm.as<int32_t>(), nullptr, nullptr, rbase.as<int32_t>(),
                                                         S.recs.as<int4>(), S.gdst.as<int32_t>());
            SPMM_CUDA(cudaGetLastError());
        } else {
            n_fgroups = 0;
        }
    }
    const int32_t fr = S.fuse;
    if (fr == 1) {
        k_segment_counts<<<g1(n_long + 1), 256, 0, s>>>(lpos.as<int32_t>(), n_long, ps.as<int32_t>(), n_short, rowptr,
                                                        split, rpw, tasks.as<int32_t>(), groups.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
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
        if (fr > 1) {
            if (n_fgroups > 0)
                k_fill_fused<<<g1(n_fgroups), 256, 0, s>>>(gseg.as<int32_t>(), n_fgroups, gbase.as<int32_t>(),
                                                           ngroups.as<int32_t>(), taskbase.as<int32_t>(),
                                                           ucnt.as<int32_t>(), rbase.as<int32_t>(), rpw, win,
                                                           S.units.as<int4>());
        } else {
            DevBuf slen;
            SPMM_TRY(slen.alloc(std::max(n_short, 1) * sizeof(int32_t), s));
            k_short_len<<<g1(M), 256, 0, s>>>(fs.as<int32_t>(), ps.as<int32_t>(), rowptr, M, slen.as<int32_t>());
            k_fill_short<<<g1(M), 256, 0, s>>>(fs.as<int32_t>(), ps.as<int32_t>(), pl.as<int32_t>(), lpos.as<int32_t>(),
                                               taskbase.as<int32_t>(), rowptr, h->perm.as<int32_t>(), slen.as<int32_t>(),
                                               n_short, n_long, M, rpw, win, S.units.as<int4>());
        }
        if (n_long > 0)
            k_fill_long<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div((int64_t)n_long * 32, 256), 148 * 32)),
                          256, 0, s>>>(lpos.as<int32_t>(), n_long, ps.as<int32_t>(), taskbase.as<int32_t>(),
                                       S.pslot_ptr.as<int32_t>(), rowptr, h->perm.as<int32_t>(), rpw, fr,
                                       S.units.as<int4>(), S.long_dst.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    S.rpw = rpw;
    return SPMM_OK;
}

using SpmmKernel = void (*)(const int4 *, int64_t, const int2 *, const float4 *, float4 *, int32_t, int32_t, float4 *,
                            unsigned int *, const int4 *, const int32_t *, const CExtra);

// W = 4 (LDG.128) geometries: any power-of-two G <= 32, V in 1..4 (no extra-destination variants: spmm_run_to
// copies C to the extra destinations after the run on these geometries)
template <int V, bool MASK, bool MD>
SpmmKernel pick_w4(int G) {
    switch (G) {
        case 1: return k_spmm<V, 1, MASK, 4, 1, MD>;
        case 2: return k_spmm<V, 2, MASK, 4, 1, MD>;
        case 4: return k_spmm<V, 4, MASK, 4, 1, MD>;
        case 8: return k_spmm<V, 8, MASK, 4, 1, MD>;
        case 16: return k_spmm<V, 16, MASK, 4, 1, MD>;
        default: return k_spmm<V, 32, MASK, 4, 1, MD>;
    }
}
template <bool MASK, bool MD>
SpmmKernel pick_w4v(int V, int G) {
    return V == 4 ? pick_w4<4, MASK, MD>(G) : V == 3 ? pick_w4<3, MASK, MD>(G) : V == 2 ? pick_w4<2, MASK, MD>(G)
                  : pick_w4<1, MASK, MD>(G);
}
// 256-bit lane loads (W = 8), exact fits only
template <bool MD>
SpmmKernel pick_w8(int V, int G) {
    switch (V * 100 + G) {
        case 104: return k_spmm<1, 4, false, 8, 1, MD>;
        case 108: return k_spmm<1, 8, false, 8, 1, MD>;
        case 204: return k_spmm<2, 4, false, 8, 1, MD>;
        case 208: return k_spmm<2, 8, false, 8, 1, MD>;
        case 408: return k_spmm<4, 8, false, 8, 1, MD>;
        case 416: return k_spmm<4, 16, false, 8, 1, MD>;
        case 432: return k_spmm<4, 32, false, 8, 1, MD>;
        default: return nullptr;
    }
}
// Row fusion only where it measured faster: G = 8 lanes per row, K = 64 (V = 1): R = 4 rows per
// group, 4 union records per inner step; K = 128 (V = 2): R = 2, 2 records per step.  At K = 32 (G = 4) a B row is
// one 128-byte line and the 32-byte records cost as much as they save (0.199 -> 0.197 ms at C2, 0.229 ms with the
// prefetch pipeline); at K = 256 the R*V accumulators do not fit.
template <bool MD>
SpmmKernel pick_w8_fused(int V, int G) {
    switch (V * 100 + G) {
        case 108: return k_spmm<1, 8, false, 8, 4, MD>;
        case 208: return k_spmm<2, 8, false, 8, 2, MD>;
        default: return nullptr;
    }
}

struct Config {
    SpmmKernel kern;
    int V, G, tiles, W;
    SpmmKernel kern_fused = nullptr;   // the same geometry with fused tasks (nullptr: no row fusion)
    int R = 1;
};

// Lane geometry.  W = 8 (one 256-bit load per lane and vector) when K % 8 == 0 and B, C are 32-byte aligned:
// 8*V*G == K with G in {8, 4} preferred (a group's load covers whole 128-byte lines; G = 8 keeps 4 rows per
// warp at K >= 64), else G in {16, 32} with V = 4.  Otherwise W = 4: exact fit 4*V*G == K with V in
// {4,3,2,1} and G a power of two <= 32, preferring G >= 8 (G*16 B >= 128 B: an L1 wavefront per line,
// measured to halve L1 data-pipe load at K=64); else V=4 with a masked column tail.
template <bool MD>
Config choose(int32_t K4, bool w8ok) {
    if (w8ok && K4 % 2 == 0) {
        const int32_t K8 = K4 / 2;
        for (int G : {8, 4})
            for (int V : {1, 2, 4})
                if (V * G == K8) {
                    SpmmKernel k = pick_w8<MD>(V, G);
                    if (k) {
                        Config c{k, V, G, 1, 8};
                        c.kern_fused = pick_w8_fused<MD>(V, G);
                        c.R = c.kern_fused ? (V == 1 ? 4 : 2) : 1;
                        return c;
                    }
                }
        for (int G : {16, 32})
            if (4 * G == K8) return {pick_w8<MD>(4, G), 4, G, 1, 8};
    }
    for (int V = 4; V >= 1; --V) {
        if (K4 % V) continue;
        const int G = K4 / V;
        if (G >= 8 && G <= 32 && (G & (G - 1)) == 0) return {pick_w4v<false, false>(V, G), V, G, 1, 4};
    }
    for (int V = 4; V >= 1; --V) {
        if (K4 % V) continue;
        const int G = K4 / V;
        if (G >= 1 && G <= 32 && (G & (G - 1)) == 0) return {pick_w4v<false, false>(V, G), V, G, 1, 4};
    }
    int G = 1;
    while (G < 32 && 4 * G < K4) G <<= 1;
    return {pick_w4<4, true, false>(G), 4, G, (int)ceil_div(K4, 4 * G), 4};
}

Config choose_for(spmm_ctx *h, int64_t K, const float *B, const float *C, const CExtra &cx, int64_t ldc) {
    uintptr_t align = (uintptr_t)B | (uintptr_t)C | (uintptr_t)(4 * ldc);   // C rows start at C + r * ldc
    for (int i = 0; i < cx.n; ++i) align |= (uintptr_t)cx.p[i];
    const bool w8ok = K % 8 == 0 && (align % 32) == 0;
    Config cfg = cx.n > 0 ? choose<true>((int32_t)(K / 4), w8ok) : choose<false>((int32_t)(K / 4), w8ok);
    if (h->params.fuse_rows == 1) {    // row fusion off (spmm_params.fuse_rows)
        cfg.kern_fused = nullptr;
        cfg.R = 1;
    }
    return cfg;
}

}  // namespace

// The schedule for (rpw, R): a cached slot, else built into the oldest slot (waiting for this handle's runs in
// flight first, since they may read the slot being replaced).  Called with h->mu held.  allow_build = false (a run
// being captured into a CUDA graph): a missing schedule is an error, since building one synchronises.
static spmm_status get_schedule(spmm_ctx *h, int32_t rpw, int32_t R, cudaStream_t s, int *slot_out,
                                bool allow_build = true) {
    int oldest = 0;
    for (int i = 0; i < SCHED_CACHE; ++i) {
        const Schedule &S = h->sched[i];
        if (S.built && S.rpw == rpw && S.fuse_req == R) {
            *slot_out = i;
            return SPMM_OK;
        }
        if (S.built < h->sched[oldest].built) oldest = i;
    }
    if (!allow_build)
        return fail(SPMM_ERR_STATE, "no run schedule for this K: call spmm_prepare(h, K, ...) before capturing spmm_run "
                                    "into a CUDA graph");
    for (int i = 0; i < RUN_SLOTS; ++i)
        if (h->slots[i].used) SPMM_CUDA(cudaEventSynchronize(h->slots[i].done));
    Schedule &S = h->sched[oldest];
    S.built = 0;
    SPMM_TRY(build_schedule(h, S, rpw, R, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    S.built = ++h->sched_seq;
    *slot_out = oldest;
    return SPMM_OK;
}

spmm_status prepare_schedule(spmm_ctx *h, int64_t K, const float *B, const float *C, cudaStream_t s) {
    const Config cfg = choose_for(h, K, B, C, CExtra{}, K);
    std::lock_guard<std::mutex> lk(h->mu);
    int slot = 0;
    SPMM_TRY(get_schedule(h, 32 / cfg.G, cfg.R, s, &slot));
    // the scratch of runs captured into CUDA graphs (no allocation may happen inside a capture)
    RunSlot &cs = h->cap_slot;
    if (cs.counters.bytes < 64 * sizeof(unsigned int)) SPMM_TRY(cs.counters.alloc(64 * sizeof(unsigned int), s));
    const size_t need = (size_t)h->sched[slot].n_pslots * K * sizeof(float);
    if (cs.partials.bytes < need) SPMM_TRY(cs.partials.alloc(need, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    // the fused kernel's schedule falls back to R = 1 when the unions do not pay; the W = 4 geometry of the same K
    // (misaligned B / C) shares rpw only when G matches, so it is prepared on first use
    return SPMM_OK;
}

void release_run_slots(spmm_ctx *h) {
    for (int i = 0; i <= RUN_SLOTS; ++i) {
        RunSlot &r = i < RUN_SLOTS ? h->slots[i] : h->cap_slot;
        if (r.done) {
            cudaEventSynchronize(r.done);
            cudaEventDestroy(r.done);
        }
        if (r.side) {
            cudaStreamSynchronize(r.side);
            cudaStreamDestroy(r.side);
        }
        if (r.fork) cudaEventDestroy(r.fork);
        if (r.join) cudaEventDestroy(r.join);
        r.counters.release();
        r.partials.release();
        r.done = r.fork = r.join = nullptr;
        r.side = nullptr;
        r.used = false;
    }
}

spmm_status launch_spmm(spmm_ctx *h, const float *B, int64_t K, float *C, int64_t ldc, cudaStream_t s,
                        int32_t *launches, const CExtra &cx) {
    *launches = 0;
    const int64_t M = h->M;
    if (M == 0) return SPMM_OK;
    const int32_t K4 = (int32_t)(K / 4), ldc4 = (int32_t)(ldc / 4);
    Config cfg = choose_for(h, K, B, C, cx, ldc);   // (W = 8 needs 32-byte aligned rows: C and ldc)
    bool copy_extra = false;      // spmm_run_to on a geometry without a multi-destination kernel: copy afterwards
    if (cx.n > 0 && !(cfg.W == 8 && cfg.tiles == 1)) {
        if (cx.mc || cx.skip_main || ldc != K)
            return fail(SPMM_ERR_UNSUPPORTED, "multicast / strided extra destinations need K % 8 == 0 and 32-byte "
                                              "aligned B and C rows");
        cfg = choose_for(h, K, B, C, CExtra{}, ldc);
        copy_extra = true;
    }
    const int32_t rpw = 32 / cfg.G;
    // a run being captured into a CUDA graph (cudaStreamBeginCapture / torch.cuda.graph) uses the handle's capture
    // slot: no host synchronisation, no allocation, no wait on events recorded outside the capture -- its schedule and
    // scratch come from spmm_prepare.  Replays of graphs capturing runs of one handle must be ordered (one stream).
    cudaStreamCaptureStatus cst = cudaStreamCaptureStatusNone;
    SPMM_CUDA(cudaStreamIsCapturing(s, &cst));
    const bool capturing = cst != cudaStreamCaptureStatusNone;
    RunSlot *rs = nullptr;
    int sidx = 0;
    {
        std::lock_guard<std::mutex> lk(h->mu);
        SPMM_TRY(get_schedule(h, rpw, cfg.R, s, &sidx, !capturing));
        rs = capturing ? &h->cap_slot : &h->slots[h->next_slot++ % RUN_SLOTS];
        if (!rs->done) {
            SPMM_CUDA(cudaEventCreateWithFlags(&rs->done, cudaEventDisableTiming));
            SPMM_CUDA(cudaStreamCreateWithFlags(&rs->side, cudaStreamNonBlocking));
            SPMM_CUDA(cudaEventCreateWithFlags(&rs->fork, cudaEventDisableTiming));
            SPMM_CUDA(cudaEventCreateWithFlags(&rs->join, cudaEventDisableTiming));
        }
        // the slot's previous run (maybe on another stream) must be done with its scratch
        if (rs->used && !capturing) SPMM_CUDA(cudaStreamWaitEvent(s, rs->done, 0));
        rs->used = !capturing;
        h->last_sched.store(sidx);
    }
    const Schedule &S = h->sched[sidx];
    const SpmmKernel kern = S.fuse > 1 ? cfg.kern_fused : cfg.kern;
    float4 *C4 = reinterpret_cast<float4 *>(C);
    float4 *P4 = nullptr;
    if (S.n_pslots > 0) {
        const size_t need = (size_t)S.n_pslots * K * sizeof(float);
        if (rs->partials.bytes < need) {
            if (capturing) return fail(SPMM_ERR_STATE, "capture: call spmm_prepare with this K first (scratch)");
            SPMM_TRY(rs->partials.alloc(need, s));
        }
        P4 = rs->partials.as<float4>();
    }
    // empty rows: zero fill on the slot's side stream forked from / joined to `s`, one small CTA per SM, so its HBM
    // writes run alongside the L2-bound SpMM kernel (measured 2-4 % faster steps than a preceding launch).  Its width
    // follows the share of the step it has to hide under: 1 warp per SM when the empty rows' bytes are a small
    // fraction of the SpMM's B-row gather bytes (C3 / C5: 1.5-2 %; a faster fill there only competes with the SpMM's
    // own DRAM traffic: C5 k_spmm +4 %), up to 4 when they are large (the last C5 shard at 8 GPUs: 8 %, where the
    // narrow fill outlasted the SpMM: shard step 4.0 -> 2.5 ms).
    bool joined = true;
    if (S.n_empty > 0) {
        const double zero_bytes = (double)S.n_empty * K * 4.0;
        const double gather_bytes = std::max(1.0, (double)(h->nnz) * K * 4.0);
        const int zw = (int)std::min(4.0, std::max(1.0, std::ceil(50.0 * zero_bytes / gather_bytes)));
        SPMM_CUDA(cudaEventRecord(rs->fork, s));
        SPMM_CUDA(cudaStreamWaitEvent(rs->side, rs->fork, 0));
        k_zero_rows<<<(unsigned)h->num_sms, 32 * zw, 0, rs->side>>>(S.empty_dst.as<int32_t>(), S.n_empty, K4, ldc4, C4,
                                                                copy_extra ? CExtra{} : cx);
        SPMM_CUDA(cudaGetLastError());
        SPMM_CUDA(cudaEventRecord(rs->join, rs->side));
        joined = false;
        ++*launches;
    }
    if (S.n_tasks > 0) {
        int occ = 0;
        SPMM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, SPMM_THREADS, 0));
        occ = std::max(occ, 1);
        const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(S.n_tasks, SPMM_THREADS / 32),
                                                                      (int64_t)h->num_sms * occ));
        const dim3 grid((unsigned)blocks, (unsigned)cfg.tiles);
        if (rs->counters.bytes < (size_t)cfg.tiles * sizeof(unsigned int)) {
            if (capturing) return fail(SPMM_ERR_STATE, "capture: call spmm_prepare with this K first (scratch)");
            SPMM_TRY(rs->counters.alloc(64 * sizeof(unsigned int), s));
        }
        SPMM_CUDA(cudaMemsetAsync(rs->counters.p, 0, (size_t)cfg.tiles * sizeof(unsigned int), s));
        const bool timed = h->timing && !capturing;
        if (timed) SPMM_CUDA(cudaEventRecord(h->ev0, s));
        kern<<<grid, SPMM_THREADS, 0, s>>>(S.units.as<int4>(), S.n_tasks, h->cv_p.as<int2>(),
                                           reinterpret_cast<const float4 *>(B), C4, K4, ldc4, P4,
                                           rs->counters.as<unsigned int>(), S.recs.as<int4>(), S.gdst.as<int32_t>(),
                                           copy_extra ? CExtra{} : cx);
        SPMM_CUDA(cudaGetLastError());
        if (timed) {
            SPMM_CUDA(cudaEventRecord(h->ev1, s));
            h->timed = true;
        }
        ++*launches;
    }
    if (S.n_long > 0) {
        k_combine<<<(unsigned)std::min<int64_t>(ceil_div(S.n_long, 8), 148 * 64), 256, 0, s>>>(
            P4, S.pslot_ptr.as<int32_t>(), S.long_dst.as<int32_t>(), S.n_long, C4, K4, ldc4,
            copy_extra ? CExtra{} : cx);
        SPMM_CUDA(cudaGetLastError());
        ++*launches;
    }
    if (!joined) SPMM_CUDA(cudaStreamWaitEvent(s, rs->join, 0));
    if (copy_extra)
        for (int i = 0; i < cx.n; ++i)
            SPMM_CUDA(cudaMemcpyAsync(cx.p[i], C, (size_t)M * K * sizeof(float), cudaMemcpyDeviceToDevice, s));
    if (!capturing) SPMM_CUDA(cudaEventRecord(rs->done, s));
    return SPMM_OK;
}

}  // namespace spmm
