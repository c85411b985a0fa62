// permute.cu -- device builders for the row permutations of PAPER.md §III and the
// permuted CSR they imply ("preserve the CSR representation").
//
//   a2 row keys (K1)          nnz_i, warp load wl_i = ceil(nnz_i/nt)            (§II.C)
//   a3 load-balance orders    NNZ_SORT / PLAIN_SORT: stable radix sort, desc key (reading A1-A3)
//                             FLIPPED, LPT (reading A5), DCSR
//   a4 signatures (K3)        blocks_i = sorted unique col/bw
//   a5 locality orders (K4)   windowed greedy chains, one CTA per window/segment: CTA_AWARE,
//                             HYBRID_1, HYBRID_2_1/2_2, WARP_AWARE,
//                             HYBRID_2_3; Hamming = |a|+|b|-2|a∩b| with the reference row's
//                             blocks held as a bitmap in shared memory ("Hamming distance (XOR)")
//   a6 permuted CSR (K5)      rowptr' = scan(nnz[perm]), (col,val) segments gathered, interleaved int2
//   a7 long-row chunks (K6)   rows with nnz > split_nnz cut into split_nnz chunks
// Every argmin is over a total order ending in the original row id, so the result is deterministic
// and bit-identical to the oracle (DESIGN.md §"Readings").
#include "internal.cuh"
#include <type_traits>
#include <algorithm>
#include <cstdlib>
#include <vector>

namespace spmm {
namespace {

__global__ void k_iota(int32_t *p, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = (int32_t)i;
}

__global__ void k_row_nnz(const int32_t *rowidx, int64_t M, int32_t *nnz) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x)
        nnz[i] = rowidx[i + 1] - rowidx[i];
}

// sort keys: ascending (maxkey - key) == descending key; value = row id (stable => ties by id)
__global__ void k_sort_keys(const int32_t *nnz, int64_t M, int32_t nt, int use_wl, int32_t maxkey, uint64_t *keys,
                            uint32_t *vals) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t k = use_wl ? (nnz[i] + nt - 1) / nt : nnz[i];
        keys[i] = (uint64_t)(maxkey - k);
        vals[i] = (uint32_t)i;
    }
}

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

// MinHash pre-order key h_i = min_{b in blocks_i} splitmix64(b ^ seed); empty -> 2^64-1 (warp per row)
__global__ void k_minhash(const int32_t *sig_ptr, const int32_t *sig, int64_t M, uint64_t seed, uint64_t *keys,
                          uint32_t *vals) {
    const int lane = threadIdx.x & 31;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < M;
         i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        uint64_t m = ~0ULL;
        for (int32_t t = sig_ptr[i] + lane; t < sig_ptr[i + 1]; t += 32)
            m = min(m, splitmix64((uint64_t)(uint32_t)sig[t] ^ seed));
#pragma unroll
        for (int o = 16; o; o >>= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
        if (lane == 0) { keys[i] = m; vals[i] = (uint32_t)i; }
    }
}

// median-block pre-order key (preorder = 2): the lower median of the row's sorted distinct blocks; empty rows last
__global__ void k_median_block(const int32_t *sig_ptr, const int32_t *sig, int64_t M, uint64_t *keys, uint32_t *vals) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t a = sig_ptr[i], n = sig_ptr[i + 1] - a;
        keys[i] = n > 0 ? (uint64_t)(uint32_t)sig[a + (n - 1) / 2] : ~0ULL;
        vals[i] = (uint32_t)i;
    }
}

// ---- signatures: warp per row; distinct blocks are the positions where col/bw changes ---------
__global__ void k_sig_count(const int32_t *rowidx, const int32_t *colidx, int64_t M, int32_t bw, int32_t *cnt) {
    const int lane = threadIdx.x & 31;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < M;
         i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        int32_t a = rowidx[i], b = rowidx[i + 1], c = 0;
        for (int32_t j = a + lane; j < b; j += 32)
            c += (j == a) || (colidx[j] / bw != colidx[j - 1] / bw);
#pragma unroll
        for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
        if (lane == 0) cnt[i] = c;
    }
}

__global__ void k_sig_fill(const int32_t *rowidx, const int32_t *colidx, int64_t M, int32_t bw, const int32_t *ptr,
                           int32_t *blk) {
    const int lane = threadIdx.x & 31;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < M;
         i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        int32_t a = rowidx[i], b = rowidx[i + 1], w = ptr[i];
        for (int32_t j0 = a; j0 < b; j0 += 32) {
            int32_t j = j0 + lane;
            bool f = j < b && ((j == a) || (colidx[j] / bw != colidx[j - 1] / bw));
            unsigned m = __ballot_sync(0xffffffffu, f);
            if (f) blk[w + __popc(m & ((1u << lane) - 1u))] = colidx[j] / bw;
            w += __popc(m);
        }
    }
}

// ---- greedy chains --------------------------------------------------------------------------
enum ChainMode { C_CTA = 0, C_H21 = 1, C_H22 = 2, C_H1 = 3, C_WARP = 4, C_H23 = 5 };
constexpr int CHAIN_THREADS = 512;
constexpr int CHAIN_MAX_PER_THREAD = 64;                 // placed flags in one u64 per thread
constexpr int64_t CHAIN_MAX_N = (int64_t)CHAIN_THREADS * CHAIN_MAX_PER_THREAD;   // 32768

struct Key {
    uint32_t k1, k2, r, a;
};
__device__ __forceinline__ bool key_less(const Key &x, const Key &y) {
    if (x.k1 != y.k1) return x.k1 < y.k1;
    if (x.k2 != y.k2) return x.k2 < y.k2;
    return x.r < y.r;
}
__device__ __forceinline__ Key shfl_key(const Key &k, int o) {
    Key y;
    y.k1 = __shfl_xor_sync(0xffffffffu, k.k1, o);
    y.k2 = __shfl_xor_sync(0xffffffffu, k.k2, o);
    y.r = __shfl_xor_sync(0xffffffffu, k.r, o);
    y.a = __shfl_xor_sync(0xffffffffu, k.a, o);
    return y;
}

// block-wide argmin; every thread returns the winner.  Uses red[] (CHAIN_THREADS/32 entries).
__device__ __forceinline__ Key block_argmin(Key k, Key *red) {
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        Key y = shfl_key(k, o);
        if (key_less(y, k)) k = y;
    }
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = k;
    __syncthreads();
    Key b = red[0];
#pragma unroll
    for (int w = 1; w < CHAIN_THREADS / 32; ++w)
        if (key_less(red[w], b)) b = red[w];
    return b;
}

__device__ __forceinline__ void bitmap_set(uint32_t *bm, const int32_t *sig, int32_t s0, int32_t s1) {
    for (int32_t t = s0 + threadIdx.x; t < s1; t += CHAIN_THREADS) {
        uint32_t b = (uint32_t)sig[t];
        atomicOr(&bm[b >> 5], 1u << (b & 31));
    }
}
__device__ __forceinline__ void bitmap_clear(uint32_t *bm, const int32_t *sig, int32_t s0, int32_t s1) {
    for (int32_t t = s0 + threadIdx.x; t < s1; t += CHAIN_THREADS) bm[(uint32_t)sig[t] >> 5] = 0u;
}
__device__ __forceinline__ uint32_t intersect(const uint32_t *bm, const int32_t *sig, int32_t s0, int32_t s1) {
    uint32_t c = 0;
    for (int32_t t = s0; t < s1; ++t) {
        uint32_t b = (uint32_t)__ldg(sig + t);
        c += (bm[b >> 5] >> (b & 31)) & 1u;
    }
    return c;
}

// One CTA per segment.  base: row ids in pre-order; segment s = base[seg[s] .. seg[s+1]) (or fixed
// windows of W when seg == nullptr).  Writes perm[seg[s] + q] for q = 0..n-1.
// Per step: (1) set the reference row's blocks in a bitmap, barrier; (2) every thread scores its
// unplaced candidates (Hamming = |ref| + |r| - 2|ref ∩ r|), block argmin (one more barrier);
// (3) clear the bitmap.  Bitmaps and the reduction buffer are double-buffered so two barriers per
// step suffice: a buffer written at step q is next written at step q+2.
template <int MODE>
__global__ void __launch_bounds__(CHAIN_THREADS) k_chain(const int32_t *base, const int32_t *seg, int64_t W, int64_t M,
                                                         const int32_t *sig_ptr, const int32_t *sig,
                                                         const int32_t *nnz, int32_t nt, int32_t nw, int64_t words,
                                                         uint32_t *gscratch, int32_t *perm) {
    extern __shared__ uint32_t smem_bm[];
    __shared__ Key red[2][CHAIN_THREADS / 32];
    constexpr int REFS = (MODE == C_H22) ? 2 : 1;   // bitmaps per step
    uint32_t *bm = gscratch ? gscratch + (size_t)blockIdx.x * 2 * REFS * words : smem_bm;
    const int64_t s0 = seg ? seg[blockIdx.x] : (int64_t)blockIdx.x * W;
    const int64_t s1 = seg ? seg[blockIdx.x + 1] : min(s0 + W, M);
    const int n = (int)(s1 - s0);
    const int32_t *om = base + s0;
    int32_t *out = perm + s0;
    for (int64_t t = threadIdx.x; t < 2 * REFS * words; t += CHAIN_THREADS) bm[t] = 0u;
    uint64_t placed = 0;   // bit k: candidate a = threadIdx.x + k*CHAIN_THREADS is placed
    __syncthreads();

    auto wl_of = [&](int32_t r) -> uint32_t { return (uint32_t)((nnz[r] + nt - 1) / nt); };
    int32_t prev = -1;
    int q = 0;
    int nfirst;
    if (MODE == C_H1) {               // Hybrid-1: the segment's first (Plain-Sort) row stays first
        nfirst = 0;
        if (n > 0) {
            if (threadIdx.x == 0) { placed |= 1ULL; out[0] = om[0]; }
            prev = om[0];
            q = 1;
        }
    } else {                          // lowest (wl, id) first: 1 row (CTA-aware), nw rows (Warp-aware)
        nfirst = (MODE == C_WARP || MODE == C_H23) ? min(n, nw) : min(n, 1);
    }
    for (; q < n; ++q) {
        const int buf = q & 1;
        const bool first = q < nfirst;
        uint32_t *bmA = bm + (size_t)(buf * REFS) * words;
        uint32_t *bmB = bmA + words;   // H22 only
        int32_t refA = -1, refB = -1;
        if (!first) {
            if (MODE == C_WARP || MODE == C_H23) refA = nw == 1 ? prev : out[q - nw];
            else refA = prev;
            if (MODE == C_H22 && q >= nw) refB = nw == 1 ? prev : out[q - nw];
        }
        int32_t aS = 0, aE = 0, bS = 0, bE = 0;
        if (refA >= 0) { aS = sig_ptr[refA]; aE = sig_ptr[refA + 1]; bitmap_set(bmA, sig, aS, aE); }
        if (refB >= 0) { bS = sig_ptr[refB]; bE = sig_ptr[refB + 1]; bitmap_set(bmB, sig, bS, bE); }
        const uint32_t cntA = (uint32_t)(aE - aS), cntB = (uint32_t)(bE - bS);
        const uint32_t wl_prev = ((MODE == C_H21 || MODE == C_H23) && !first) ? wl_of(prev) : 0u;
        __syncthreads();
        Key best{0xffffffffu, 0xffffffffu, 0xffffffffu, 0xffffffffu};
        for (int k = 0; k < CHAIN_MAX_PER_THREAD; ++k) {
            const int a = threadIdx.x + k * CHAIN_THREADS;
            if (a >= n) break;
            if ((placed >> k) & 1ULL) continue;
            const int32_t r = om[a];
            Key c{0u, 0u, (uint32_t)r, (uint32_t)a};
            if (first) {
                c.k1 = wl_of(r);
            } else {
                const int32_t rs = sig_ptr[r], re = sig_ptr[r + 1];
                const uint32_t cr = (uint32_t)(re - rs);
                c.k1 = cntA + cr - 2u * intersect(bmA, sig, rs, re);
                if (MODE == C_H21 || MODE == C_H23) {
                    const uint32_t w = wl_of(r);
                    c.k2 = w > wl_prev ? w - wl_prev : wl_prev - w;
                } else if (MODE == C_H22) {
                    c.k2 = refB >= 0 ? cntB + cr - 2u * intersect(bmB, sig, rs, re) : 0u;
                }
            }
            if (key_less(c, best)) best = c;
        }
        const Key w = block_argmin(best, red[buf]);
        if ((int)(w.a % CHAIN_THREADS) == (int)threadIdx.x) placed |= 1ULL << (w.a / CHAIN_THREADS);
        if (threadIdx.x == 0) out[q] = (int32_t)w.r;
        if (refA >= 0) bitmap_clear(bmA, sig, aS, aE);
        if (refB >= 0) bitmap_clear(bmB, sig, bS, bE);
        prev = (int32_t)w.r;
    }
}

// HYBRID_1 segments: p starts a segment if it starts a run of equal sorted key or is W positions
// into its run.  keys: ascending sorted (maxwl - wl).
__global__ void k_h1_flags(const uint64_t *keys, int64_t M, int64_t W, int32_t *flag) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        // run start = lower_bound(keys, keys[p])
        int64_t lo = 0, hi = p;
        uint64_t k = keys[p];
        while (lo < hi) {
            int64_t mid = (lo + hi) >> 1;
            if (keys[mid] < k) lo = mid + 1; else hi = mid;
        }
        flag[p] = ((p - lo) % W) == 0;
    }
}

__global__ void k_compact_starts(const int32_t *flag, const int32_t *pos, int64_t M, int32_t *starts) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x)
        if (flag[p]) starts[pos[p]] = (int32_t)p;
}

__global__ void k_set_last(int32_t *a, int64_t idx, int32_t v) { a[idx] = v; }

// FLIPPED: odd nw-chunks of the Plain-Sort order reversed (a partial last chunk within its length)
__global__ void k_flip(const uint32_t *s, int64_t M, int32_t nw, int32_t *perm) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = p / nw, lo = c * nw, hi = min(lo + nw, M);
        perm[p] = (int32_t)((c & 1) ? s[lo + (hi - 1 - p)] : s[p]);
    }
}

// LPT (capacity-constrained, reading A5): one warp; lane w holds warp w's load / count / capacity.
__global__ void k_lpt(const uint32_t *s, const int32_t *nnz, int64_t M, int32_t nt, int32_t nw, int32_t *perm) {
    const int lane = threadIdx.x;
    int64_t load = 0, cnt = 0;
    const int64_t cap = (lane < nw && M > lane) ? (M - lane + nw - 1) / nw : 0;
    for (int64_t t0 = 0; t0 < M; t0 += 32) {
        int64_t t = t0 + lane;
        uint32_t r_mine = t < M ? s[t] : 0u;
        int32_t wl_mine = t < M ? (nnz[r_mine] + nt - 1) / nt : 0;
        int lim = (int)(M - t0 < 32 ? M - t0 : 32);
        for (int u = 0; u < lim; ++u) {
            uint32_t r = __shfl_sync(0xffffffffu, r_mine, u);
            int32_t wl = __shfl_sync(0xffffffffu, wl_mine, u);
            // argmin over non-full warps of (load, w)
            int64_t key_load = (lane < nw && cnt < cap) ? load : INT64_MAX;
            int key_w = lane;
#pragma unroll
            for (int o = 16; o; o >>= 1) {
                int64_t ol = __shfl_xor_sync(0xffffffffu, key_load, o);
                int ow = __shfl_xor_sync(0xffffffffu, key_w, o);
                if (ol < key_load || (ol == key_load && ow < key_w)) { key_load = ol; key_w = ow; }
            }
            if (lane == key_w) {
                perm[cnt * nw + lane] = (int32_t)r;
                load += wl;
                ++cnt;
            }
        }
    }
}

__global__ void k_dcsr_flags(const int32_t *nnz, int64_t M, int32_t *flag) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x)
        flag[i] = nnz[i] > 0;
}
__global__ void k_dcsr_scatter(const int32_t *flag, const int32_t *pos, int64_t M, int32_t n_nonempty, int32_t *perm) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x)
        perm[flag[i] ? pos[i] : n_nonempty + ((int32_t)i - pos[i])] = (int32_t)i;
}

__global__ void k_u32_to_i32(const uint32_t *a, int64_t n, int32_t *b) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        b[i] = (int32_t)a[i];
}

// ---- permuted CSR ---------------------------------------------------------------------------
__global__ void k_perm_len(const int32_t *rowidx, const int32_t *perm, int64_t M, int32_t *len) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        int32_t i = perm[p];
        len[p] = rowidx[i + 1] - rowidx[i];
    }
}

// warp per position: copy the row's (col, val) pairs into the interleaved permuted array
__global__ void k_gather(const int32_t *rowidx, const int32_t *colidx, const float *value, const int32_t *perm,
                         const int32_t *rowptr_p, int64_t M, int2 *cv) {
    const int lane = threadIdx.x & 31;
    for (int64_t p = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; p < M;
         p += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        int32_t i = perm[p];
        int32_t a = rowidx[i], len = rowidx[i + 1] - a, d = rowptr_p[p];
        for (int32_t t = lane; t < len; t += 32)
            cv[d + t] = make_int2(colidx[a + t], __float_as_int(value[a + t]));
    }
}

__global__ void k_long_flags(const int32_t *rowptr_p, int64_t M, int32_t split, int32_t *flag, int32_t *nch) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x) {
        int32_t len = rowptr_p[p + 1] - rowptr_p[p];
        bool lg = len > split;
        flag[p] = lg;
        nch[p] = lg ? (len + split - 1) / split : 0;
    }
}

inline unsigned grid_for(int64_t n, int threads) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, threads), 148 * 32));
}
inline unsigned grid_warps(int64_t n, int threads) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n * 32, threads), 148 * 64));
}

spmm_status launch_chain(int mode, const int32_t *base, const int32_t *seg, int64_t nseg, int64_t W, int64_t M,
                         const Signatures &sig, const int32_t *nnz, const spmm_params &p, int64_t N, int32_t *perm,
                         cudaStream_t s) {
    if (nseg == 0) return SPMM_OK;
    const int64_t nblk = ceil_div(N, p.bw);
    const int64_t words = std::max<int64_t>(1, ceil_div(nblk, 32));
    const int nbuf = mode == C_H22 ? 4 : 2;   // 2 buffers x refs
    size_t smem = (size_t)nbuf * words * sizeof(uint32_t);
    DevBuf gs;
    uint32_t *gscratch = nullptr;
    if (smem > 200 * 1024) {   // large N: per-CTA bitmaps in global memory (L2-resident)
        SPMM_TRY(gs.alloc((size_t)nseg * nbuf * words * sizeof(uint32_t), s));
        gscratch = gs.as<uint32_t>();
        smem = 0;
    }
    auto go = [&](auto kern) -> spmm_status {
        if (smem > 48 * 1024) SPMM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        kern<<<(unsigned)nseg, CHAIN_THREADS, smem, s>>>(base, seg, W, M, sig.ptr.as<int32_t>(), sig.blk.as<int32_t>(),
                                                        nnz, p.nt, p.nw, words, gscratch, perm);
        SPMM_CUDA(cudaGetLastError());
        return SPMM_OK;
    };
    switch (mode) {
        case C_CTA: return go(k_chain<C_CTA>);
        case C_H21: return go(k_chain<C_H21>);
        case C_H22: return go(k_chain<C_H22>);
        case C_H1: return go(k_chain<C_H1>);
        case C_WARP: return go(k_chain<C_WARP>);
        default: return go(k_chain<C_H23>);
    }
}

// ---- paper-exact chains over windows above 32768 rows, up to W = M (f3) -----------
// The same definitions as k_chain (CTA_AWARE: next = argmin over the window's unplaced rows of
// (ham(r, prev), r); HYBRID_2_1: (ham, |wl_r - wl_prev|, r)), evaluated through an
// inverted index block -> rows instead of scoring every candidate each step:
//   ham(r, prev) = |b_prev| + |b_r| - 2 |b_r ∩ b_prev|, and a row sharing no block with prev scores
//   |b_prev| + |b_r|.  So the argmin lies in T ∪ {u*}: T = the unplaced rows of prev's posting lists
//   (scored exactly, |b_r ∩ b_prev| counted by one atomic per list entry), u* = the best untouched-form
//   candidate: the unplaced row of least (|b|, r) (CTA_AWARE) or, among the unplaced rows of the least
//   |b| = b0, the least (|wl - wl_prev|, r) (HYBRID_2_1).  Any row outside T scores >= u* under the key
//   (DESIGN.md §6 "exact chains"), so the result is the definition's, bit-identical to k_chain / oracle.
// One CTA of 1024 threads per window; per step: count pass, barrier, score pass, block argmin.  The
// counters are double-buffered by step parity and the previous step's lists are zeroed during the
// count pass, so they need no pass of their own.
constexpr int XCH_THREADS = 1024;
constexpr int XCH_CACHE = XCH_THREADS;   // posting-list prefix of up to 1024 blocks kept in smem per step
constexpr int XT_CAP = 8192;             // k_chain_x: touched rows listed per step (dynamic smem, 2 buffers)
#ifdef SPMM_EXP_NO_XT   // A/B variant: no touched list in k_chain_x (score and reset re-walk the posting lists)
constexpr int32_t XT_USE = -1;
#else
constexpr int32_t XT_USE = XT_CAP;
#endif

__global__ void k_win_of(const int32_t *base, int64_t M, int64_t W, int32_t *win) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < M; q += (int64_t)gridDim.x * blockDim.x)
        win[base[q]] = (int32_t)(q / W);
}
__global__ void k_win_of_seg(const int32_t *base, const int32_t *seg, int64_t nseg, int64_t M, int32_t *win) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < M; q += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = 0, hi = nseg - 1;              // last segment with seg[k] <= q
        while (lo < hi) {
            const int64_t mid = (lo + hi + 1) >> 1;
            if (seg[mid] <= q) lo = mid;
            else hi = mid - 1;
        }
        win[base[q]] = (int32_t)lo;
    }
}
__global__ void k_blk_count(const int32_t *blk, int64_t S, int32_t *bcnt) {
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < S; t += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(&bcnt[blk[t]], 1);
}
__global__ void k_blk_fill(const int32_t *sig_ptr, const int32_t *blk, int64_t M, const int32_t *bptr, int32_t *bcur,
                           int32_t *brow) {
    const int lane = threadIdx.x & 31;
    for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < M;
         r += ((int64_t)gridDim.x * blockDim.x) >> 5)
        for (int32_t t = sig_ptr[r] + lane; t < sig_ptr[r + 1]; t += 32) {
            const int32_t b = blk[t];
            brow[bptr[b] + atomicAdd(&bcur[b], 1)] = (int32_t)r;
        }
}
// multi-window: posting entries keyed by (window of the row, block), so a window's posting lists are one contiguous
// chunk, list by list (rows ascending within a list: the sort is stable over entries in row order); the values are
// the entry ids t, the entry's row goes to erow[t]
__global__ void k_blk_win_keys(const int32_t *sig_ptr, const int32_t *blk, int64_t M, const int32_t *win, int bb,
                               uint64_t *keys, uint32_t *vals, int32_t *erow) {
    const int lane = threadIdx.x & 31;
    for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < M;
         r += ((int64_t)gridDim.x * blockDim.x) >> 5)
        for (int32_t t = sig_ptr[r] + lane; t < sig_ptr[r + 1]; t += 32) {
            keys[t] = ((uint64_t)(uint32_t)win[r] << bb) | (uint32_t)blk[t];
            vals[t] = (uint32_t)t;
            erow[t] = (int32_t)r;
        }
}
// runs of equal (window, block) keys = the window sub-lists: flag[i] = 1 at the first entry of a run
__global__ void k_run_flags(const uint64_t *keys, int64_t S, int32_t *flag) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < S; i += (int64_t)gridDim.x * blockDim.x)
        flag[i] = (i == 0 || keys[i] != keys[i - 1]) ? 1 : 0;
}
__global__ void k_run_starts(const int32_t *flag, const int32_t *pos, int64_t S, int32_t *rstart) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < S; i += (int64_t)gridDim.x * blockDim.x)
        if (flag[i]) rstart[pos[i]] = (int32_t)i;
}
// per sorted entry i (entry id e = vals[i]): xr[e] = its run [start, end), brow[i] = its row
__global__ void k_xr_fill(const uint32_t *vals, const int32_t *flag, const int32_t *pos, const int32_t *rstart,
                          const int32_t *erow, int64_t S, int2 *xr, int32_t *brow) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < S; i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t e = vals[i];
        const int32_t rid = pos[i] + flag[i] - 1;
        xr[e] = make_int2(rstart[rid], rstart[rid + 1]);
        brow[i] = erow[e];
    }
}
__global__ void k_xkeys(const int32_t *sig_ptr, const int32_t *nnz, int64_t M, int32_t nt, int with_wl, uint64_t *keys,
                        uint32_t *vals) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < M; r += (int64_t)gridDim.x * blockDim.x) {
        const uint64_t nb = (uint64_t)(sig_ptr[r + 1] - sig_ptr[r]);
        const uint64_t wl = (uint64_t)((nnz[r] + nt - 1) / nt);
        keys[r] = with_wl ? (nb << 26) | wl : nb;
        vals[r] = (uint32_t)r;
    }
}
__global__ void k_xkeys_win(const uint32_t *vals, const int32_t *win, int64_t M, uint64_t *keys) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x)
        keys[i] = (uint64_t)win[vals[i]];
}

__device__ __forceinline__ bool is_placed(const uint32_t *placed, int32_t r) {
    return (__ldcg(placed + (r >> 5)) >> (r & 31)) & 1u;
}

// block-wide argmin over XCH_THREADS threads; every thread returns the winner
__device__ __forceinline__ Key xblock_argmin(Key k, Key *red) {
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        Key y = shfl_key(k, o);
        if (key_less(y, k)) k = y;
    }
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = k;
    __syncthreads();
    Key b = red[threadIdx.x & 31];
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        Key y = shfl_key(b, o);
        if (key_less(y, b)) b = y;
    }
    return b;
}

// prefix of the posting-list lengths of blocks sig_blk[c0 .. c0+nb) into pre[0..nb], list starts into bst[]
// mwin >= 0 (multi-window): only the window's sub-range of each list, xr[entry] = [start, end) (k_xr_fill)
template <class PT>
__device__ __forceinline__ void xprefix(const int32_t *sig_blk, const int32_t *bptr, int32_t c0, int32_t nb,
                                        PT *pre, int32_t *bst, PT *wsum, const int32_t *brow = nullptr,
                                        const int32_t *win = nullptr, int32_t mwin = -1,
                                        const int2 *xr = nullptr) {
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    int32_t len = 0;
    if (tid < nb) {
        int32_t a, e;
        if (mwin >= 0) {                        // the window's sub-range of the list (k_xr_fill)
            const int2 v = __ldg(xr + c0 + tid);
            a = v.x;
            e = v.y;
        } else {
            const int32_t b = sig_blk[c0 + tid];
            a = bptr[b];
            e = bptr[b + 1];
        }
        len = e - a;
        bst[tid] = a;
    }
    PT x = len;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const PT y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[wid] = x;
    __syncthreads();
    // every warp scans the 32 warp totals itself (one barrier fewer than a warp-0 scan + broadcast)
    PT w = wsum[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const PT y = __shfl_up_sync(0xffffffffu, w, o);
        if (lane >= o) w += y;
    }
    const PT off = __shfl_sync(0xffffffffu, w, (wid + 31) & 31);
    pre[tid + 1] = x + (wid ? off : 0);
    if (tid == 0) pre[0] = 0;
    __syncthreads();
}

// visit every entry of the posting lists described by (pre, bst, nb): f(row)
// PT: prefix type -- int32 when 1024 x the longest posting list fits (the host checks), else int64
template <class PT, class IT, class F>
__device__ __forceinline__ void xvisit(const PT *pre, const int32_t *bst, int32_t nb, const IT *brow, F f) {
    const PT T = pre[nb];
    for (PT e = threadIdx.x; e < T; e += XCH_THREADS) {
        int lo = 0, hi = nb - 1;
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (pre[mid] <= e) lo = mid;
            else hi = mid - 1;
        }
        f((int32_t)__ldg(brow + bst[lo] + (e - pre[lo])));
    }
}

// all entries of row r0's lists, chunked by XCH_THREADS blocks (re-derives the prefix; barriers inside)
// IT = int32_t: brow holds row ids (and serves the binary searches when xr is NULL); IT = uint16_t: window-local
// row indices (k_chain_xl, xr required)
template <class PT, class IT, class F>
__device__ __forceinline__ void xvisit_all(int32_t r0, const int32_t *sig_ptr, const int32_t *sig_blk,
                                           const int32_t *bptr, const IT *brow, PT *pre, int32_t *bst,
                                           PT *wsum, const int32_t *win, int32_t mwin, const int2 *xr, F f) {
    const int32_t bs = sig_ptr[r0], be = sig_ptr[r0 + 1];
    for (int32_t c0 = bs; c0 < be; c0 += XCH_THREADS) {
        const int32_t nb = min(XCH_THREADS, be - c0);
        xprefix(sig_blk, bptr, c0, nb, pre, bst, wsum,
                std::is_same<IT, int32_t>::value ? reinterpret_cast<const int32_t *>(brow) : nullptr, win, mwin, xr);
        xvisit(pre, bst, nb, brow, f);
        __syncthreads();
    }
}

template <int MODE, class PT>
__global__ void __launch_bounds__(XCH_THREADS, 1) k_chain_x(const int32_t *base, const int32_t *seg, int64_t W,
                                                            int64_t M, int multiwin,
                                                            const int32_t *sig_ptr, const int32_t *sig_blk,
                                                            const int32_t *bptr, const int32_t *brow,
                                                            const int32_t *win, const int2 *xr, const uint32_t *ord,
                                                            const int32_t *nnz, int32_t nt, int32_t nw,
                                                            uint32_t *placed, int32_t *cnt0, int32_t *cnt1,
                                                            int32_t *cnt2a, int32_t *cnt2b, int32_t *perm) {
    // HYBRID_2_2: key (ham(r, prev), q >= nw ? ham(r, out[q - nw]) : 0, r) -- a second reference ref2
    // with its own counters (cnt2a/b) and scratch; the argmin lies in T1 ∪ (T2 ∩ class b0) ∪ {u*}
    constexpr bool TWOREF = MODE == C_H22;
    constexpr int C2 = TWOREF ? XCH_CACHE : 1;
    __shared__ PT pre2[C2 + 1];
    __shared__ int32_t bst2[C2];
    __shared__ PT pre[2][XCH_CACHE + 1];
    __shared__ int32_t bst[2][XCH_CACHE];
    __shared__ PT wsum[32];
    __shared__ Key red[2][XCH_THREADS / 32];
    __shared__ int32_t s_ptr;
    // the distinct rows a step's count pass touched (its T; up to XT_CAP, listed on first touch): the score pass and
    // the next step's counter reset walk it instead of re-walking the posting lists (re-walk when it overflowed)
    extern __shared__ int32_t xt_s[];   // [2][XT_CAP]
    __shared__ int32_t s_nt[2];
    const int32_t w = (int32_t)blockIdx.x;
    // window w = positions [s0, s1) of the pre-order: fixed windows of W, or HYBRID_1's segments (seg)
    const int64_t s0 = seg ? seg[w] : (int64_t)w * W, s1 = seg ? seg[w + 1] : min(s0 + W, M);
    const int32_t n = (int32_t)(s1 - s0);
    const uint32_t *o = ord + s0;            // the window's rows by (|b|, [wl,] r)
    int32_t *out = perm + s0;
    auto nb_of = [&](int32_t r) -> uint32_t { return (uint32_t)(sig_ptr[r + 1] - sig_ptr[r]); };
    auto wl_of = [&](int32_t r) -> uint32_t { return (uint32_t)((nnz[r] + nt - 1) / nt); };
    // multi-window: lists are sorted by window and only this window's sub-range is visited, so every row a
    // pass sees belongs to this window (and only this CTA touches its counters)
    const int32_t mw = multiwin ? w : -1;
    if (n <= 0) return;
    // first row(s): least (wl, r) of the window's unplaced rows -- 1 row (CTA_AWARE, HYBRID_2_1), nw rows
    // (WARP_AWARE, HYBRID_2_3: "the first 32 rows are those ... with the lowest warp load"), as k_chain
    // (HYBRID_1: every row of a segment has the same wl and the segment lists them in ascending id, so its
    //  least (wl, r) is its first row -- the row P:L132 / reading A8 starts the segment with)
    constexpr bool WARPREF = MODE == C_WARP || MODE == C_H23;   // Hamming reference out[q - nw], else prev
    const int32_t nfirst = WARPREF ? min(n, nw) : 1;
    Key best;
    int32_t prev = -1, pprev = -1, pref = -1, pref2 = -1;
    if (threadIdx.x < 2) s_nt[threadIdx.x] = 0;   // ordered by the first rows' barriers
    for (int32_t q = 0; q < nfirst; ++q) {
        best = Key{0xffffffffu, 0xffffffffu, 0xffffffffu, 0u};
        for (int32_t a = threadIdx.x; a < n; a += XCH_THREADS) {
            const int32_t r = base[s0 + a];
            if (q > 0 && is_placed(placed, r)) continue;
            Key c{wl_of(r), 0u, (uint32_t)r, 0u};
            if (key_less(c, best)) best = c;
        }
        const Key w0 = xblock_argmin(best, red[q & 1]);
        prev = (int32_t)w0.r;
        if (threadIdx.x == 0) {
            out[q] = prev;
            atomicOr(placed + (prev >> 5), 1u << (prev & 31));
            s_ptr = 0;
        }
        __syncthreads();
    }
    bool cached_pp = false;
    for (int32_t q = nfirst; q < n; ++q) {
        const int buf = q & 1;
        int32_t *cc = buf ? cnt1 : cnt0, *co = buf ? cnt0 : cnt1;
        int32_t *xt = xt_s + buf * XT_CAP;
        const int32_t *xto = xt_s + (buf ^ 1) * XT_CAP;
        const int32_t nto = s_nt[buf ^ 1];   // the previous step's touched count (> XT_CAP: overflowed)
        __syncthreads();                     // everyone has read s_nt[buf ^ 1] / s_nt[buf] of earlier steps
        if (threadIdx.x == 0) s_nt[buf] = 0;
        // the row Hamming distances are taken to; out[q - 1] is written by thread 0 after the previous step's
        // last barrier, so nw == 1 reads it from the register copy prev (as k_chain does)
        const int32_t ref = WARPREF ? (nw == 1 ? prev : out[q - nw]) : prev;
        const int32_t bs = sig_ptr[ref], be = sig_ptr[ref + 1];
        const uint32_t cp = (uint32_t)(be - bs);
        const bool cached = be - bs <= XCH_CACHE;
        // prefix of ref's lists (kept for the score pass and for the next step's reset); the previous
        // step's prefix lives in the other buffer
        if (cached) xprefix(sig_blk, bptr, bs, be - bs, pre[buf], bst[buf], wsum, brow, win, mw, xr);
        // reset the previous step's counters (other buffer), then count |b_r ∩ b_ref|
        if (pref >= 0 && nto <= XT_USE) {
            for (int32_t i = threadIdx.x; i < nto; i += XCH_THREADS) co[xto[i]] = 0;
        } else if (pref >= 0) {
            auto reset = [&](int32_t r) { co[r] = 0; };
            if (cached_pp) xvisit(pre[buf ^ 1], bst[buf ^ 1], sig_ptr[pref + 1] - sig_ptr[pref], brow, reset);
            else xvisit_all(pref, sig_ptr, sig_blk, bptr, brow, pre[buf ^ 1], bst[buf ^ 1], wsum, win, mw, xr, reset);
        }
        auto count = [&](int32_t r) {
            if (r != prev && !is_placed(placed, r) && atomicAdd(cc + r, 1) == 0) {
                const int32_t i = atomicAdd(&s_nt[buf], 1);
                if (i < XT_USE) xt[i] = r;
            }
        };
        if (cached) xvisit(pre[buf], bst[buf], be - bs, brow, count);
        else xvisit_all(ref, sig_ptr, sig_blk, bptr, brow, pre[buf], bst[buf], wsum, win, mw, xr, count);
        int32_t ref2 = -1;
        int32_t *cc2 = buf ? cnt2b : cnt2a;
        uint32_t cp2 = 0;
        if constexpr (TWOREF) {
            int32_t *co2 = buf ? cnt2a : cnt2b;
            if (pref2 >= 0)
                xvisit_all(pref2, sig_ptr, sig_blk, bptr, brow, pre2, bst2, wsum, win, mw, xr, [&](int32_t r) { co2[r] = 0; });
            ref2 = q >= nw ? (nw == 1 ? prev : out[q - nw]) : -1;
            if (ref2 >= 0) {
                cp2 = nb_of(ref2);
                xvisit_all(ref2, sig_ptr, sig_blk, bptr, brow, pre2, bst2, wsum, win, mw, xr, [&](int32_t r) {
                    if (r != prev && !is_placed(placed, r)) atomicAdd(cc2 + r, 1);
                });
            }
        }
        __syncthreads();
        constexpr bool WLTIE = MODE == C_H21 || MODE == C_H23;      // tie: |wl_r - wl_prev|
        const uint32_t wlp = WLTIE ? wl_of(prev) : 0u;
        auto keyof = [&](int32_t r) -> Key {
            const uint32_t c = (uint32_t)__ldcg(cc + r);
            Key k{cp + nb_of(r) - 2u * c, 0u, (uint32_t)r, 0u};
            if (WLTIE) {
                const uint32_t x = wl_of(r);
                k.k2 = x > wlp ? x - wlp : wlp - x;
            }
            if (TWOREF && ref2 >= 0) k.k2 = cp2 + nb_of(r) - 2u * (uint32_t)__ldcg(cc2 + r);
            return k;
        };
        best = Key{0xffffffffu, 0xffffffffu, 0xffffffffu, 0u};
        auto score = [&](int32_t r) {
            if (r != prev && !is_placed(placed, r)) {
                const Key k = keyof(r);
                if (key_less(k, best)) best = k;
            }
        };
        const int32_t nt1 = s_nt[buf];
        if (nt1 <= XT_USE) for (int32_t i = threadIdx.x; i < nt1; i += XCH_THREADS) score(xt[i]);
        else if (cached) xvisit(pre[buf], bst[buf], be - bs, brow, score);
        else xvisit_all(ref, sig_ptr, sig_blk, bptr, brow, pre[buf], bst[buf], wsum, win, mw, xr, score);
        if constexpr (TWOREF) {
            if (ref2 >= 0) {
                // T2 ∩ class b0: b0 = |b| of the first unplaced row of the (|b|, r) order
                if (threadIdx.x < 32) {
                    const int lane = threadIdx.x;
                    int32_t ptr = s_ptr;
                    while (ptr < n) {
                        const bool pl = ptr + lane < n ? is_placed(placed, (int32_t)o[ptr + lane]) : false;
                        const unsigned m = __ballot_sync(0xffffffffu, !pl && ptr + lane < n);
                        if (m) { ptr += __ffs(m) - 1; break; }
                        ptr = min(ptr + 32, n);
                    }
                    __syncwarp();
                    if (lane == 0) s_ptr = ptr;
                }
                __syncthreads();
                const int32_t ptr = s_ptr;
                const uint32_t b0 = ptr < n ? nb_of((int32_t)o[ptr]) : 0xffffffffu;
                __syncthreads();   // everyone has read s_ptr before warp 0 may rewrite it below
                xvisit_all(ref2, sig_ptr, sig_blk, bptr, brow, pre2, bst2, wsum, win, mw, xr, [&](int32_t r) {
                    if (r != prev && !is_placed(placed, r) && nb_of(r) == b0) {
                        const Key k = keyof(r);
                        if (key_less(k, best)) best = k;
                    }
                });
            }
        }
        // u*: the first unplaced row of the (|b|, [wl,] r) order (placed rows before s_ptr stay placed)
        if (threadIdx.x < 32) {
            const int lane = threadIdx.x;
            int32_t ptr = s_ptr;
            while (ptr < n) {   // warp-wide skip over placed entries, 32 at a time
                const bool pl = ptr + lane < n ? is_placed(placed, (int32_t)o[ptr + lane]) : false;
                const unsigned m = __ballot_sync(0xffffffffu, !pl && ptr + lane < n);
                if (m) { ptr += __ffs(m) - 1; break; }
                ptr = min(ptr + 32, n);
            }
            __syncwarp();
            if (lane == 0) s_ptr = ptr;
            if (ptr < n) {
                if (!WLTIE) {
                    if (lane == 0) {
                        const Key k = keyof((int32_t)o[ptr]);
                        if (key_less(k, best)) best = k;
                    }
                } else {
                    // class b0 = |b| of o[ptr]; inside it rows are ordered by (wl, r)
                    const uint32_t b0 = nb_of((int32_t)o[ptr]);
                    int32_t lo = ptr, hi = n;                     // class end: first index with |b| > b0
                    while (lo < hi) { const int32_t mid = (lo + hi) >> 1; if (nb_of((int32_t)o[mid]) > b0) hi = mid; else lo = mid + 1; }
                    const int32_t cend = lo;
                    lo = ptr; hi = cend;                          // lb: first index with wl >= wl_prev
                    while (lo < hi) { const int32_t mid = (lo + hi) >> 1; if (wl_of((int32_t)o[mid]) >= wlp) hi = mid; else lo = mid + 1; }
                    const int32_t lb = lo;
                    // up: first unplaced in [lb, cend)
                    for (int32_t i = lb; i < cend; i += 32) {
                        const bool ok = i + lane < cend && !is_placed(placed, (int32_t)o[i + lane]);
                        const unsigned m = __ballot_sync(0xffffffffu, ok);
                        if (m) {
                            if (lane == 0) {
                                const Key k = keyof((int32_t)o[i + __ffs(m) - 1]);
                                if (key_less(k, best)) best = k;
                            }
                            break;
                        }
                    }
                    // down: last unplaced in [ptr, lb), then the first unplaced of its wl run
                    int32_t d = -1;
                    for (int32_t i = lb - 1; i >= ptr; i -= 32) {
                        const bool ok = i - lane >= ptr && !is_placed(placed, (int32_t)o[i - lane]);
                        const unsigned m = __ballot_sync(0xffffffffu, ok);
                        if (m) { d = i - (__ffs(m) - 1); break; }
                    }
                    if (d >= 0) {
                        const uint32_t wd = wl_of((int32_t)o[d]);
                        lo = ptr; hi = d;
                        while (lo < hi) { const int32_t mid = (lo + hi) >> 1; if (wl_of((int32_t)o[mid]) >= wd) hi = mid; else lo = mid + 1; }
                        for (int32_t i = lo; i <= d; i += 32) {
                            const bool ok = i + lane <= d && !is_placed(placed, (int32_t)o[i + lane]);
                            const unsigned m = __ballot_sync(0xffffffffu, ok);
                            if (m) {
                                if (lane == 0) {
                                    const Key k = keyof((int32_t)o[i + __ffs(m) - 1]);
                                    if (key_less(k, best)) best = k;
                                }
                                break;
                            }
                        }
                    }
                }
            }
        }
        const Key nx = xblock_argmin(best, red[buf]);
        if (threadIdx.x == 0) {
            out[q] = (int32_t)nx.r;
            atomicOr(placed + (nx.r >> 5), 1u << (nx.r & 31));
        }
        pprev = prev;
        pref = ref;
        pref2 = ref2;
        cached_pp = cached;
        prev = (int32_t)nx.r;
    }
}

// k_chain_xl: k_chain_x for windows of at most XL_MAX rows (every windowed chain policy) with the
// window held in shared memory.  The posting-list entries carry the row's index inside its window (bloc, 16 bit),
// so the per-step state -- the |b_r ∩ b_ref| counters, the placed flags, |b_r|, wl_r, the row ids and the
// (|b|, [wl,] r) order -- is indexed locally: the count pass is a shared-memory atomic, the score pass and the u*
// search read shared memory, where k_chain_x makes global atomics and L2 round trips on every step's critical path.
// Same definitions, same keys, same argmin as k_chain_x (DESIGN.md §6 "exact chains"): bit-identical permutations.
constexpr int XL_MAX = 4096;
// r, nb, wl, o (u32), cnt[2] (i32), placed bits, touched lists[2] (u16)
constexpr size_t XL_SMEM = (size_t)XL_MAX * (4 * 4 + 2 * 4) + XL_MAX / 8 + (size_t)XL_MAX * 2 * 2;
// HYBRID_2_2's second reference: counters[2] (i32) and touched lists[2] (u16)
constexpr size_t XL_SMEM_H22 = XL_SMEM + (size_t)XL_MAX * (2 * 4 + 2 * 2);

__global__ void k_lpos(const int32_t *base, const int32_t *seg, int64_t W, int64_t M, const int32_t *win,
                       int32_t *lpos) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < M; q += (int64_t)gridDim.x * blockDim.x) {
        const int32_t r = base[q], w = win[r];
        lpos[r] = (int32_t)(q - (seg ? (int64_t)seg[w] : (int64_t)w * W));
    }
}
__global__ void k_bloc(const int32_t *brow, int64_t S, const int32_t *lpos, uint16_t *bloc) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < S; i += (int64_t)gridDim.x * blockDim.x)
        bloc[i] = (uint16_t)lpos[brow[i]];
}

template <int MODE, class PT>
__global__ void __launch_bounds__(XCH_THREADS, 1) k_chain_xl(const int32_t *base, const int32_t *seg, int64_t W,
                                                             int64_t M, const int32_t *sig_ptr,
                                                             const int32_t *sig_blk, const int32_t *bptr,
                                                             const uint16_t *bloc, const int2 *xr,
                                                             const uint32_t *ord, const int32_t *lpos,
                                                             const int32_t *nnz, int32_t nt, int32_t nw,
                                                             int32_t *perm) {
    extern __shared__ uint32_t xl[];
    __shared__ PT pre[2][XCH_CACHE + 1];
    __shared__ int32_t bst[2][XCH_CACHE];
    __shared__ PT wsum[32];
    __shared__ Key red[2][XCH_THREADS / 32];
    __shared__ int32_t s_ptr;
    // HYBRID_2_2: key (ham(r, prev), q >= nw ? ham(r, out[q - nw]) : 0, r) -- a second reference ref2 with
    // its own counters and touched list; the argmin lies in T1 ∪ (T2 ∩ class b0) ∪ {u*}
    constexpr bool TWOREF = MODE == C_H22;
    constexpr int C2 = TWOREF ? XCH_CACHE : 1;
    __shared__ PT pre2[C2 + 1];
    __shared__ int32_t bst2[C2];
    __shared__ int32_t s_nt2[2];
    const int32_t w = (int32_t)blockIdx.x;
    const int64_t s0 = seg ? seg[w] : (int64_t)w * W, s1 = seg ? seg[w + 1] : min(s0 + W, M);
    const int32_t n = (int32_t)(s1 - s0);
    if (n <= 0) return;
    int32_t *r_s = reinterpret_cast<int32_t *>(xl);           // local index -> row id
    uint32_t *nb_s = xl + XL_MAX;                            // |b_r|
    uint32_t *wl_s = xl + 2 * XL_MAX;                        // wl_r
    uint32_t *o_s = xl + 3 * XL_MAX;                         // the window's (|b|, [wl,] r) order, local indices
    int32_t *cnt_s = reinterpret_cast<int32_t *>(xl + 4 * XL_MAX);   // [2][XL_MAX] counters by step parity
    uint32_t *pl_s = xl + 6 * XL_MAX;                        // placed flags
    // the distinct rows a step's count pass touched (its candidate set T, listed on first touch): the score pass
    // and the next step's counter reset walk this list instead of re-walking the posting lists
    uint16_t *tl_s = reinterpret_cast<uint16_t *>(pl_s + XL_MAX / 32);   // [2][XL_MAX]
    __shared__ int32_t s_nt[2];
    int32_t *cnt2_s = reinterpret_cast<int32_t *>(tl_s + 2 * XL_MAX);   // [2][XL_MAX] (HYBRID_2_2 only)
    uint16_t *tl2_s = reinterpret_cast<uint16_t *>(cnt2_s + 2 * XL_MAX);  // [2][XL_MAX] (HYBRID_2_2 only)
    for (int32_t a = threadIdx.x; a < n; a += XCH_THREADS) {
        const int32_t r = base[s0 + a];
        r_s[a] = r;
        nb_s[a] = (uint32_t)(sig_ptr[r + 1] - sig_ptr[r]);
        wl_s[a] = (uint32_t)((nnz[r] + nt - 1) / nt);
        o_s[a] = (uint32_t)lpos[ord[s0 + a]];
        cnt_s[a] = 0;
        cnt_s[XL_MAX + a] = 0;
        if (TWOREF) {
            cnt2_s[a] = 0;
            cnt2_s[XL_MAX + a] = 0;
        }
    }
    for (int32_t a = threadIdx.x; a < (n + 31) / 32; a += XCH_THREADS) pl_s[a] = 0u;
    if (threadIdx.x < 2) s_nt[threadIdx.x] = s_nt2[threadIdx.x] = 0;
    __syncthreads();
    auto placed = [&](int32_t l) -> bool { return (pl_s[l >> 5] >> (l & 31)) & 1u; };
    int32_t *out = perm + s0;
    constexpr bool WARPREF = MODE == C_WARP || MODE == C_H23;   // Hamming reference out[q - nw], else prev
    constexpr bool WLTIE = MODE == C_H21 || MODE == C_H23;      // tie: |wl_r - wl_prev|
    const int32_t nfirst = WARPREF ? min(n, nw) : 1;
    Key best;
    int32_t prev = -1, prev_l = -1;
    for (int32_t q = 0; q < nfirst; ++q) {
        best = Key{0xffffffffu, 0xffffffffu, 0xffffffffu, 0u};
        for (int32_t a = threadIdx.x; a < n; a += XCH_THREADS) {
            if (q > 0 && placed(a)) continue;
            const Key c{wl_s[a], 0u, (uint32_t)r_s[a], (uint32_t)a};
            if (key_less(c, best)) best = c;
        }
        const Key w0 = xblock_argmin(best, red[q & 1]);
        prev = (int32_t)w0.r;
        prev_l = (int32_t)w0.a;
        if (threadIdx.x == 0) {
            out[q] = prev;
            pl_s[prev_l >> 5] |= 1u << (prev_l & 31);
            s_ptr = 0;
        }
        __syncthreads();
    }
    for (int32_t q = nfirst; q < n; ++q) {
        const int buf = q & 1;
        int32_t *cc = cnt_s + buf * XL_MAX, *co = cnt_s + (buf ^ 1) * XL_MAX;
        const int32_t ref = WARPREF ? (nw == 1 ? prev : out[q - nw]) : prev;
        const int32_t bs = sig_ptr[ref], be = sig_ptr[ref + 1];
        const uint32_t cp = (uint32_t)(be - bs);
        const bool cached = be - bs <= XCH_CACHE;
        uint16_t *tl = tl_s + buf * XL_MAX, *tlo = tl_s + (buf ^ 1) * XL_MAX;
        // the previous step's touched rows: reset their counters (other buffer); this step's list restarts (every
        // reader of s_nt[buf] -- step q-1's reset -- is behind the barriers of step q-1's passes)
        for (int32_t i = threadIdx.x; i < s_nt[buf ^ 1]; i += XCH_THREADS) co[tlo[i]] = 0;
        if (threadIdx.x == 0) s_nt[buf] = 0;   // ordered before the count pass by xprefix's barriers
        int32_t *cc2 = cnt2_s + buf * XL_MAX;
        uint16_t *tl2 = tl2_s + buf * XL_MAX;
        if constexpr (TWOREF) {
            int32_t *co2 = cnt2_s + (buf ^ 1) * XL_MAX;
            const uint16_t *tl2o = tl2_s + (buf ^ 1) * XL_MAX;
            for (int32_t i = threadIdx.x; i < s_nt2[buf ^ 1]; i += XCH_THREADS) co2[tl2o[i]] = 0;
            if (threadIdx.x == 0) s_nt2[buf] = 0;
        }
        if (cached) xprefix(sig_blk, bptr, bs, be - bs, pre[buf], bst[buf], wsum, nullptr, nullptr, w, xr);
        auto count = [&](int32_t l) {
            if (l != prev_l && !placed(l) && atomicAdd(cc + l, 1) == 0) tl[atomicAdd(&s_nt[buf], 1)] = (uint16_t)l;
        };
        if (cached) xvisit(pre[buf], bst[buf], be - bs, bloc, count);
        else xvisit_all(ref, sig_ptr, sig_blk, bptr, bloc, pre[buf], bst[buf], wsum, nullptr, w, xr, count);
        int32_t ref2 = -1;
        uint32_t cp2 = 0;
        if constexpr (TWOREF) {
            ref2 = q >= nw ? (nw == 1 ? prev : out[q - nw]) : -1;
            if (ref2 >= 0) {
                cp2 = (uint32_t)(sig_ptr[ref2 + 1] - sig_ptr[ref2]);
                __syncthreads();   // pre2 / bst2 / wsum of a previous pass are free (xvisit_all re-derives them)
                xvisit_all(ref2, sig_ptr, sig_blk, bptr, bloc, pre2, bst2, wsum, nullptr, w, xr, [&](int32_t l) {
                    if (l != prev_l && !placed(l) && atomicAdd(cc2 + l, 1) == 0)
                        tl2[atomicAdd(&s_nt2[buf], 1)] = (uint16_t)l;
                });
            }
        }
        __syncthreads();
        const uint32_t wlp = WLTIE ? wl_s[prev_l] : 0u;
        auto keyof = [&](int32_t l) -> Key {
            Key k{cp + nb_s[l] - 2u * (uint32_t)cc[l], 0u, (uint32_t)r_s[l], (uint32_t)l};
            if (WLTIE) {
                const uint32_t x = wl_s[l];
                k.k2 = x > wlp ? x - wlp : wlp - x;
            }
            if (TWOREF && ref2 >= 0) k.k2 = cp2 + nb_s[l] - 2u * (uint32_t)cc2[l];
            return k;
        };
        best = Key{0xffffffffu, 0xffffffffu, 0xffffffffu, 0u};
        auto score = [&](int32_t l) {
            if (l != prev_l && !placed(l)) {
                const Key k = keyof(l);
                if (key_less(k, best)) best = k;
            }
        };
        for (int32_t i = threadIdx.x; i < s_nt[buf]; i += XCH_THREADS) score((int32_t)tl[i]);
        if constexpr (TWOREF) {
            if (ref2 >= 0) {
                // T2 ∩ class b0: b0 = |b| of the first unplaced row of the (|b|, r) order
                if (threadIdx.x < 32) {
                    const int lane = threadIdx.x;
                    int32_t ptr = s_ptr;
                    while (ptr < n) {
                        const bool pl = ptr + lane < n ? placed((int32_t)o_s[ptr + lane]) : false;
                        const unsigned m = __ballot_sync(0xffffffffu, !pl && ptr + lane < n);
                        if (m) { ptr += __ffs(m) - 1; break; }
                        ptr = min(ptr + 32, n);
                    }
                    __syncwarp();
                    if (lane == 0) s_ptr = ptr;
                }
                __syncthreads();
                const int32_t ptr = s_ptr;
                const uint32_t b0 = ptr < n ? nb_s[o_s[ptr]] : 0xffffffffu;
                __syncthreads();   // everyone has read s_ptr before warp 0 may rewrite it below
                for (int32_t i = threadIdx.x; i < s_nt2[buf]; i += XCH_THREADS) {
                    const int32_t l = (int32_t)tl2[i];
                    if (l != prev_l && !placed(l) && nb_s[l] == b0) {
                        const Key k = keyof(l);
                        if (key_less(k, best)) best = k;
                    }
                }
            }
        }
        // u*: the first unplaced row of the (|b|, [wl,] r) order (placed rows before s_ptr stay placed)
        if (threadIdx.x < 32) {
            const int lane = threadIdx.x;
            int32_t ptr = s_ptr;
            while (ptr < n) {
                const bool pl = ptr + lane < n ? placed((int32_t)o_s[ptr + lane]) : false;
                const unsigned m = __ballot_sync(0xffffffffu, !pl && ptr + lane < n);
                if (m) { ptr += __ffs(m) - 1; break; }
                ptr = min(ptr + 32, n);
            }
            __syncwarp();
            if (lane == 0) s_ptr = ptr;
            if (ptr < n) {
                if (!WLTIE) {
                    if (lane == 0) {
                        const Key k = keyof((int32_t)o_s[ptr]);
                        if (key_less(k, best)) best = k;
                    }
                } else {
                    const uint32_t b0 = nb_s[o_s[ptr]];
                    int32_t lo = ptr, hi = n;                     // class end: first index with |b| > b0
                    while (lo < hi) { const int32_t mid = (lo + hi) >> 1; if (nb_s[o_s[mid]] > b0) hi = mid; else lo = mid + 1; }
                    const int32_t cend = lo;
                    lo = ptr; hi = cend;                          // lb: first index with wl >= wl_prev
                    while (lo < hi) { const int32_t mid = (lo + hi) >> 1; if (wl_s[o_s[mid]] >= wlp) hi = mid; else lo = mid + 1; }
                    const int32_t lb = lo;
                    for (int32_t i = lb; i < cend; i += 32) {      // up: first unplaced in [lb, cend)
                        const bool ok = i + lane < cend && !placed((int32_t)o_s[i + lane]);
                        const unsigned m = __ballot_sync(0xffffffffu, ok);
                        if (m) {
                            if (lane == 0) {
                                const Key k = keyof((int32_t)o_s[i + __ffs(m) - 1]);
                                if (key_less(k, best)) best = k;
                            }
                            break;
                        }
                    }
                    int32_t d = -1;                               // down: last unplaced in [ptr, lb)
                    for (int32_t i = lb - 1; i >= ptr; i -= 32) {
                        const bool ok = i - lane >= ptr && !placed((int32_t)o_s[i - lane]);
                        const unsigned m = __ballot_sync(0xffffffffu, ok);
                        if (m) { d = i - (__ffs(m) - 1); break; }
                    }
                    if (d >= 0) {                                 // then the first unplaced of its wl run
                        const uint32_t wd = wl_s[o_s[d]];
                        lo = ptr; hi = d;
                        while (lo < hi) { const int32_t mid = (lo + hi) >> 1; if (wl_s[o_s[mid]] >= wd) hi = mid; else lo = mid + 1; }
                        for (int32_t i = lo; i <= d; i += 32) {
                            const bool ok = i + lane <= d && !placed((int32_t)o_s[i + lane]);
                            const unsigned m = __ballot_sync(0xffffffffu, ok);
                            if (m) {
                                if (lane == 0) {
                                    const Key k = keyof((int32_t)o_s[i + __ffs(m) - 1]);
                                    if (key_less(k, best)) best = k;
                                }
                                break;
                            }
                        }
                    }
                }
            }
        }
        const Key nx = xblock_argmin(best, red[buf]);
        if (threadIdx.x == 0) {
            out[q] = (int32_t)nx.r;
            pl_s[nx.a >> 5] |= 1u << (nx.a & 31);
        }
        prev = (int32_t)nx.r;
        prev_l = (int32_t)nx.a;
    }
}

// seg != nullptr: HYBRID_1's nseg segments (positions seg[k] .. seg[k+1]) instead of windows of W
spmm_status launch_chain_exact(int mode, const int32_t *base, const int32_t *seg, int64_t nseg, int64_t W, int64_t M,
                               const Signatures &sig, const int32_t *nnz, const spmm_params &p, int64_t N,
                               int32_t *perm, cudaStream_t s) {
    const int64_t nblk = ceil_div(N, p.bw);
    const int64_t nwin = seg ? nseg : ceil_div(M, W);
    DevBuf win, bcnt, bptr, bcur, brow, keys, ord, placed, cnt;
    SPMM_TRY(win.alloc(M * sizeof(int32_t), s));
    if (seg) k_win_of_seg<<<grid_for(M, 256), 256, 0, s>>>(base, seg, nseg, M, win.as<int32_t>());
    else k_win_of<<<grid_for(M, 256), 256, 0, s>>>(base, M, W, win.as<int32_t>());
    SPMM_CUDA(cudaGetLastError());
    // inverted index: block -> rows (CSR over blocks)
    SPMM_TRY(bcnt.alloc((nblk + 1) * sizeof(int32_t), s));
    SPMM_TRY(bptr.alloc((nblk + 1) * sizeof(int32_t), s));
    SPMM_TRY(bcur.alloc((nblk + 1) * sizeof(int32_t), s));
    SPMM_CUDA(cudaMemsetAsync(bcnt.p, 0, (nblk + 1) * sizeof(int32_t), s));
    SPMM_CUDA(cudaMemsetAsync(bcur.p, 0, (nblk + 1) * sizeof(int32_t), s));
    if (sig.S > 0) {
        k_blk_count<<<grid_for(sig.S, 256), 256, 0, s>>>(sig.blk.as<int32_t>(), sig.S, bcnt.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    SPMM_TRY(exclusive_scan_i32(bcnt.as<int32_t>(), bptr.as<int32_t>(), nblk, nullptr, s));   // bptr[nblk] = S
    SPMM_TRY(brow.alloc(std::max<int64_t>(sig.S, 1) * sizeof(int32_t), s));
    DevBuf xr;
    if (sig.S > 0 && nwin > 1) {
        DevBuf ek, vals, erow, flag, pos, rstart;
        SPMM_TRY(ek.alloc(sig.S * sizeof(uint64_t), s));
        SPMM_TRY(vals.alloc(sig.S * sizeof(uint32_t), s));
        SPMM_TRY(erow.alloc(sig.S * sizeof(int32_t), s));
        int bb = 0, wb = 0;
        while (bb < 32 && ((uint64_t)nblk >> bb) != 0) ++bb;
        while (wb < 32 && ((uint64_t)nwin >> wb) != 0) ++wb;
        k_blk_win_keys<<<grid_warps(M, 256), 256, 0, s>>>(sig.ptr.as<int32_t>(), sig.blk.as<int32_t>(), M,
                                                          win.as<int32_t>(), bb, ek.as<uint64_t>(),
                                                          vals.as<uint32_t>(), erow.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(radix_sort_pairs(ek.as<uint64_t>(), vals.as<uint32_t>(), sig.S, 0, bb + wb, s));
        SPMM_TRY(flag.alloc(sig.S * sizeof(int32_t), s));
        SPMM_TRY(pos.alloc((sig.S + 1) * sizeof(int32_t), s));
        k_run_flags<<<grid_for(sig.S, 256), 256, 0, s>>>(ek.as<uint64_t>(), sig.S, flag.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        int32_t nruns = 0;
        SPMM_TRY(exclusive_scan_i32(flag.as<int32_t>(), pos.as<int32_t>(), sig.S, &nruns, s));
        SPMM_TRY(rstart.alloc(((int64_t)nruns + 1) * sizeof(int32_t), s));
        k_run_starts<<<grid_for(sig.S, 256), 256, 0, s>>>(flag.as<int32_t>(), pos.as<int32_t>(), sig.S,
                                                          rstart.as<int32_t>());
        k_set_last<<<1, 1, 0, s>>>(rstart.as<int32_t>(), nruns, (int32_t)sig.S);
        SPMM_TRY(xr.alloc(sig.S * sizeof(int2), s));
        k_xr_fill<<<grid_for(sig.S, 256), 256, 0, s>>>(vals.as<uint32_t>(), flag.as<int32_t>(), pos.as<int32_t>(),
                                                       rstart.as<int32_t>(), erow.as<int32_t>(), sig.S,
                                                       xr.as<int2>(), brow.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    } else if (sig.S > 0) {
        k_blk_fill<<<grid_warps(M, 256), 256, 0, s>>>(sig.ptr.as<int32_t>(), sig.blk.as<int32_t>(), M,
                                                      bptr.as<int32_t>(), bcur.as<int32_t>(), brow.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    // rows by (window, |b|, [wl,] r): two stable radix sorts over row ids in ascending order
    SPMM_TRY(keys.alloc(M * sizeof(uint64_t), s));
    SPMM_TRY(ord.alloc(M * sizeof(uint32_t), s));
    const bool with_wl = mode == C_H21 || mode == C_H23;
    k_xkeys<<<grid_for(M, 256), 256, 0, s>>>(sig.ptr.as<int32_t>(), nnz, M, p.nt, with_wl ? 1 : 0,
                                             keys.as<uint64_t>(), ord.as<uint32_t>());
    SPMM_CUDA(cudaGetLastError());
    SPMM_TRY(radix_sort_pairs(keys.as<uint64_t>(), ord.as<uint32_t>(), M, 0, with_wl ? 56 : 32, s));
    if (nwin > 1) {
        k_xkeys_win<<<grid_for(M, 256), 256, 0, s>>>(ord.as<uint32_t>(), win.as<int32_t>(), M, keys.as<uint64_t>());
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(radix_sort_pairs(keys.as<uint64_t>(), ord.as<uint32_t>(), M, 0, 32, s));
    }
    SPMM_TRY(placed.alloc(ceil_div(M, 32) * sizeof(uint32_t), s));
    SPMM_CUDA(cudaMemsetAsync(placed.p, 0, ceil_div(M, 32) * sizeof(uint32_t), s));
    const int64_t ncnt = mode == C_H22 ? 4 : 2;
    SPMM_TRY(cnt.alloc(ncnt * M * sizeof(int32_t), s));
    SPMM_CUDA(cudaMemsetAsync(cnt.p, 0, ncnt * M * sizeof(int32_t), s));
    // 32-bit posting-list prefixes unless 1024 x the longest list could overflow them
    int32_t max_list = 0;
    SPMM_TRY(reduce_max_i32(bcnt.as<int32_t>(), nblk, &max_list, s));
    const char *fw = getenv("SPMM_CHAIN_WIDE");   // tests: force the 64-bit variant
    const bool wide = (int64_t)max_list * XCH_CACHE >= ((int64_t)1 << 31) || (fw && atoi(fw) != 0);
    auto pick = [&](auto pt) {
        using PT = decltype(pt);
        return mode == C_H21 ? k_chain_x<C_H21, PT> : mode == C_WARP ? k_chain_x<C_WARP, PT>
             : mode == C_H23 ? k_chain_x<C_H23, PT> : mode == C_H22 ? k_chain_x<C_H22, PT>
             : k_chain_x<C_CTA, PT>;                                    // HYBRID_1 = C_CTA over segments
    };
    auto kern = wide ? pick(int64_t{}) : pick(int32_t{});
    // windows of at most XL_MAX rows (HYBRID_1's segments are cut at the window size): k_chain_xl
    const int64_t wmax = seg ? (int64_t)p.window : W;
#ifdef SPMM_EXP_NO_XL   // A/B variant: k_chain_x with global counters for every window size
    const bool local = false;
#else
    const bool local = nwin > 1 && sig.S > 0 && wmax > 0 && wmax <= XL_MAX;
#endif
    if (local) {
        DevBuf lpos, bloc;
        SPMM_TRY(lpos.alloc(M * sizeof(int32_t), s));
        SPMM_TRY(bloc.alloc(sig.S * sizeof(uint16_t), s));
        k_lpos<<<grid_for(M, 256), 256, 0, s>>>(base, seg, W, M, win.as<int32_t>(), lpos.as<int32_t>());
        k_bloc<<<grid_for(sig.S, 256), 256, 0, s>>>(brow.as<int32_t>(), sig.S, lpos.as<int32_t>(), bloc.as<uint16_t>());
        SPMM_CUDA(cudaGetLastError());
        auto pickl = [&](auto pt) {
            using PT = decltype(pt);
            return mode == C_H21 ? k_chain_xl<C_H21, PT> : mode == C_WARP ? k_chain_xl<C_WARP, PT>
                 : mode == C_H23 ? k_chain_xl<C_H23, PT> : mode == C_H22 ? k_chain_xl<C_H22, PT>
                 : k_chain_xl<C_CTA, PT>;                                   // HYBRID_1 = C_CTA
        };
        auto kl = wide ? pickl(int64_t{}) : pickl(int32_t{});
        const size_t xls = mode == C_H22 ? XL_SMEM_H22 : XL_SMEM;
        SPMM_CUDA(cudaFuncSetAttribute(kl, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)xls));
        kl<<<(unsigned)nwin, XCH_THREADS, xls, s>>>(base, seg, W, M, sig.ptr.as<int32_t>(), sig.blk.as<int32_t>(),
                                                        bptr.as<int32_t>(), bloc.as<uint16_t>(), xr.as<int2>(),
                                                        ord.as<uint32_t>(), lpos.as<int32_t>(), nnz, p.nt, p.nw, perm);
        SPMM_CUDA(cudaGetLastError());
        return SPMM_OK;
    }
    const size_t xts = 2 * XT_CAP * sizeof(int32_t);
    SPMM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)xts));
    kern<<<(unsigned)nwin, XCH_THREADS, xts, s>>>(base, seg, W, M, nwin > 1 ? 1 : 0, sig.ptr.as<int32_t>(),
                                                sig.blk.as<int32_t>(), bptr.as<int32_t>(), brow.as<int32_t>(),
                                                win.as<int32_t>(), xr.p ? xr.as<int2>() : nullptr,
                                                ord.as<uint32_t>(), nnz, p.nt, p.nw,
                                                placed.as<uint32_t>(), cnt.as<int32_t>(), cnt.as<int32_t>() + M,
                                                mode == C_H22 ? cnt.as<int32_t>() + 2 * M : nullptr,
                                                mode == C_H22 ? cnt.as<int32_t>() + 3 * M : nullptr, perm);
    SPMM_CUDA(cudaGetLastError());
    return SPMM_OK;
}

// SPMM_CHAIN_EXACT=1 / 0: force the inverted-index builder / k_chain for CTA_AWARE and HYBRID_2_1 where both
// apply (W <= 32768); unset: -1, the measured rule in build_permutation.  Read per spmm_permute call.
int force_exact_ix() {
    const char *e = getenv("SPMM_CHAIN_EXACT");
    return e && *e ? (atoi(e) != 0 ? 1 : 0) : -1;
}

// plain sort (by nnz or by warp load), result row ids in vals (uint32[M]); keys kept for H1
spmm_status sort_rows(const int32_t *nnz, int64_t M, int32_t nt, bool by_wl, int32_t max_nnz, DevBuf &keys, DevBuf &vals,
                      cudaStream_t s) {
    SPMM_TRY(keys.alloc(std::max<int64_t>(M, 1) * sizeof(uint64_t), s));
    SPMM_TRY(vals.alloc(std::max<int64_t>(M, 1) * sizeof(uint32_t), s));
    int32_t maxkey = by_wl ? (max_nnz + nt - 1) / nt : max_nnz;
    if (M == 0) return SPMM_OK;
    k_sort_keys<<<grid_for(M, 256), 256, 0, s>>>(nnz, M, nt, by_wl ? 1 : 0, maxkey, keys.as<uint64_t>(), vals.as<uint32_t>());
    SPMM_CUDA(cudaGetLastError());
    int bits = 0;
    while (bits < 32 && ((uint64_t)maxkey >> bits) != 0) ++bits;
    return radix_sort_pairs(keys.as<uint64_t>(), vals.as<uint32_t>(), M, 0, bits, s);
}

}  // namespace

spmm_status build_signatures(const int32_t *rowidx, const int32_t *colidx, const int32_t * /*order*/, int64_t M,
                             int64_t nnz, int32_t bw, Signatures &sig, cudaStream_t s) {
    DevBuf cnt;
    SPMM_TRY(cnt.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    SPMM_TRY(sig.ptr.alloc((M + 1) * sizeof(int32_t), s));
    if (M > 0) {
        k_sig_count<<<grid_warps(M, 256), 256, 0, s>>>(rowidx, colidx, M, bw, cnt.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    int32_t total = 0;
    SPMM_TRY(exclusive_scan_i32(cnt.as<int32_t>(), sig.ptr.as<int32_t>(), M, &total, s));
    sig.S = total;
    SPMM_TRY(sig.blk.alloc(std::max<int64_t>(total, 1) * sizeof(int32_t), s));
    if (M > 0 && nnz > 0) {
        k_sig_fill<<<grid_warps(M, 256), 256, 0, s>>>(rowidx, colidx, M, bw, sig.ptr.as<int32_t>(), sig.blk.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    return SPMM_OK;
}

spmm_status build_permutation(spmm_ctx *h, spmm_policy policy, const spmm_params &p, DevBuf &perm_out, cudaStream_t s) {
    const int64_t M = h->M;
    SPMM_TRY(perm_out.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    int32_t *perm = perm_out.as<int32_t>();
    if (M == 0) return SPMM_OK;
    DevBuf nnzb;
    SPMM_TRY(nnzb.alloc(M * sizeof(int32_t), s));
    int32_t *nnz = nnzb.as<int32_t>();
    k_row_nnz<<<grid_for(M, 256), 256, 0, s>>>(h->rowidx.as<int32_t>(), M, nnz);
    SPMM_CUDA(cudaGetLastError());

    switch (policy) {
    case SPMM_POLICY_IDENTITY:
        k_iota<<<grid_for(M, 256), 256, 0, s>>>(perm, M);
        SPMM_CUDA(cudaGetLastError());
        return SPMM_OK;
    case SPMM_POLICY_NNZ_SORT:
    case SPMM_POLICY_PLAIN_SORT:
    case SPMM_POLICY_FLIPPED:
    case SPMM_POLICY_LPT: {
        DevBuf keys, vals;
        SPMM_TRY(sort_rows(nnz, M, p.nt, policy != SPMM_POLICY_NNZ_SORT, h->max_row_nnz, keys, vals, s));
        if (policy == SPMM_POLICY_FLIPPED) {
            k_flip<<<grid_for(M, 256), 256, 0, s>>>(vals.as<uint32_t>(), M, p.nw, perm);
        } else if (policy == SPMM_POLICY_LPT) {
            if (p.nw > 32) return fail(SPMM_ERR_UNSUPPORTED, "LPT: nw > 32");
            k_lpt<<<1, 32, 0, s>>>(vals.as<uint32_t>(), nnz, M, p.nt, p.nw, perm);
        } else {
            k_u32_to_i32<<<grid_for(M, 256), 256, 0, s>>>(vals.as<uint32_t>(), M, perm);
        }
        SPMM_CUDA(cudaGetLastError());
        return SPMM_OK;
    }
    case SPMM_POLICY_DCSR: {
        DevBuf flag, pos;
        SPMM_TRY(flag.alloc(M * sizeof(int32_t), s));
        SPMM_TRY(pos.alloc((M + 1) * sizeof(int32_t), s));
        k_dcsr_flags<<<grid_for(M, 256), 256, 0, s>>>(nnz, M, flag.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        int32_t ne = 0;
        SPMM_TRY(exclusive_scan_i32(flag.as<int32_t>(), pos.as<int32_t>(), M, &ne, s));
        k_dcsr_scatter<<<grid_for(M, 256), 256, 0, s>>>(flag.as<int32_t>(), pos.as<int32_t>(), M, ne, perm);
        SPMM_CUDA(cudaGetLastError());
        return SPMM_OK;
    }
    case SPMM_POLICY_HYBRID_1: {
        const int64_t W = (p.window == 0 || p.window > M) ? M : p.window;
        DevBuf keys, vals, flag, pos, starts, base;
        SPMM_TRY(sort_rows(nnz, M, p.nt, true, h->max_row_nnz, keys, vals, s));
        SPMM_TRY(flag.alloc(M * sizeof(int32_t), s));
        SPMM_TRY(pos.alloc((M + 1) * sizeof(int32_t), s));
        k_h1_flags<<<grid_for(M, 256), 256, 0, s>>>(keys.as<uint64_t>(), M, W, flag.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        int32_t nseg = 0;
        SPMM_TRY(exclusive_scan_i32(flag.as<int32_t>(), pos.as<int32_t>(), M, &nseg, s));
        SPMM_TRY(starts.alloc((nseg + 1) * sizeof(int32_t), s));
        k_compact_starts<<<grid_for(M, 256), 256, 0, s>>>(flag.as<int32_t>(), pos.as<int32_t>(), M, starts.as<int32_t>());
        k_set_last<<<1, 1, 0, s>>>(starts.as<int32_t>(), nseg, (int32_t)M);
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(base.alloc(M * sizeof(int32_t), s));
        k_u32_to_i32<<<grid_for(M, 256), 256, 0, s>>>(vals.as<uint32_t>(), M, base.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
        Signatures sig;
        SPMM_TRY(build_signatures(h->rowidx.as<int32_t>(), h->colidx.as<int32_t>(), nullptr, M, h->nnz, p.bw, sig, s));
        // segments above 32768 rows (or forced, or hub rows at large W): the inverted-index builder, HYBRID_1
        // being CTA_AWARE's key over each segment (same rule as the chain policies below)
        const int fx = force_exact_ix();
        if (W > CHAIN_MAX_N || fx == 1 || (fx < 0 && (W >= 8192 || h->max_row_nnz > 1024)))
            return launch_chain_exact(C_CTA, base.as<int32_t>(), starts.as<int32_t>(), nseg, 0, M, sig, nnz, p, h->N,
                                      perm, s);
        return launch_chain(C_H1, base.as<int32_t>(), starts.as<int32_t>(), nseg, 0, M, sig, nnz, p, h->N, perm, s);
    }
    default: {   // chain policies over windows of a pre-order
        const int64_t W = (p.window == 0 || p.window > M) ? M : p.window;
        // builder choice (identical results, tests/test_gpu_exact_chains.py): k_chain scores every candidate of the
        // window each step (cost ~ W * sum of the window's signature lengths), k_chain_x walks prev's posting
        // lists; measured (profiles/r1_chain_builders.jsonl) k_chain_x wins for W >= 8192 and on inputs with hub
        // rows (C3 1024: 2.0 -> 0.55 s, C5 1024: 5.3 -> 1.9 s), k_chain on short-row inputs at small W (C2 1024:
        // 0.012 vs 0.047 s).  SPMM_CHAIN_EXACT=0 / 1 forces one builder where both apply.
        const int fx = force_exact_ix();
        const bool exact_ix = W > CHAIN_MAX_N || fx == 1 || (fx < 0 && (W >= 8192 || h->max_row_nnz > 1024));
        int mode = policy == SPMM_POLICY_CTA_AWARE ? C_CTA : policy == SPMM_POLICY_HYBRID_2_1 ? C_H21 :
                   policy == SPMM_POLICY_HYBRID_2_2 ? C_H22 : policy == SPMM_POLICY_WARP_AWARE ? C_WARP : C_H23;
        Signatures sig;
        SPMM_TRY(build_signatures(h->rowidx.as<int32_t>(), h->colidx.as<int32_t>(), nullptr, M, h->nnz, p.bw, sig, s));
        DevBuf base;
        SPMM_TRY(base.alloc(M * sizeof(int32_t), s));
        if (p.preorder) {
            DevBuf keys, vals;
            SPMM_TRY(keys.alloc(M * sizeof(uint64_t), s));
            SPMM_TRY(vals.alloc(M * sizeof(uint32_t), s));
            if (p.preorder == 2)
                k_median_block<<<grid_for(M, 256), 256, 0, s>>>(sig.ptr.as<int32_t>(), sig.blk.as<int32_t>(), M,
                                                                keys.as<uint64_t>(), vals.as<uint32_t>());
            else
                k_minhash<<<grid_warps(M, 256), 256, 0, s>>>(sig.ptr.as<int32_t>(), sig.blk.as<int32_t>(), M, p.seed,
                                                            keys.as<uint64_t>(), vals.as<uint32_t>());
            SPMM_CUDA(cudaGetLastError());
            SPMM_TRY(radix_sort_pairs(keys.as<uint64_t>(), vals.as<uint32_t>(), M, 0, 64, s));
            k_u32_to_i32<<<grid_for(M, 256), 256, 0, s>>>(vals.as<uint32_t>(), M, base.as<int32_t>());
        } else {
            k_iota<<<grid_for(M, 256), 256, 0, s>>>(base.as<int32_t>(), M);
        }
        SPMM_CUDA(cudaGetLastError());
        if (exact_ix)
            return launch_chain_exact(mode, base.as<int32_t>(), nullptr, 0, W, M, sig, nnz, p, h->N, perm, s);
        return launch_chain(mode, base.as<int32_t>(), nullptr, ceil_div(M, W), W, M, sig, nnz, p, h->N, perm, s);
    }
    }
}

spmm_status build_permuted_csr(spmm_ctx *h, int32_t split, const DevBuf &perm, DevBuf &rowptr_p, DevBuf &cv_p,
                               RowClasses &rc, cudaStream_t s) {
    const int64_t M = h->M;
    SPMM_TRY(rowptr_p.alloc((M + 1) * sizeof(int32_t), s));
    // two pairs of slack: whole 16-byte blocks of a row range can be bulk-copied without reading past the end
    SPMM_TRY(cv_p.alloc((std::max<int64_t>(h->nnz, 1) + 2) * sizeof(int2), s));
    DevBuf len;
    SPMM_TRY(len.alloc(std::max<int64_t>(M, 1) * sizeof(int32_t), s));
    if (M > 0) {
        k_perm_len<<<grid_for(M, 256), 256, 0, s>>>(h->rowidx.as<int32_t>(), perm.as<int32_t>(), M, len.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    SPMM_TRY(exclusive_scan_i32(len.as<int32_t>(), rowptr_p.as<int32_t>(), M, nullptr, s));
    if (M > 0 && h->nnz > 0) {
        k_gather<<<grid_warps(M, 256), 256, 0, s>>>(h->rowidx.as<int32_t>(), h->colidx.as<int32_t>(), h->value.as<float>(),
                                                   perm.as<int32_t>(), rowptr_p.as<int32_t>(), M, cv_p.as<int2>());
        SPMM_CUDA(cudaGetLastError());
    }
    // a7 row-class counts (the K-dependent run schedule is built by spmm_prepare / the first spmm_run)
    rc.n_long = rc.n_chunks = 0;
    if (M == 0 || h->max_row_nnz <= split) return SPMM_OK;
    DevBuf flag, nch, tmp;
    SPMM_TRY(flag.alloc(M * sizeof(int32_t), s));
    SPMM_TRY(nch.alloc(M * sizeof(int32_t), s));
    SPMM_TRY(tmp.alloc((M + 1) * sizeof(int32_t), s));
    k_long_flags<<<grid_for(M, 256), 256, 0, s>>>(rowptr_p.as<int32_t>(), M, split, flag.as<int32_t>(), nch.as<int32_t>());
    SPMM_CUDA(cudaGetLastError());
    int32_t nlong = 0, nchunks = 0;
    SPMM_TRY(exclusive_scan_i32(flag.as<int32_t>(), tmp.as<int32_t>(), M, &nlong, s));
    SPMM_TRY(exclusive_scan_i32(nch.as<int32_t>(), tmp.as<int32_t>(), M, &nchunks, s));
    rc.n_long = nlong;
    rc.n_chunks = nchunks;
    return SPMM_OK;
}

}  // namespace spmm
