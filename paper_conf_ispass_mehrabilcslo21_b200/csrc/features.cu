// features.cu -- the 24 sparsity features of Table II (§V.A) on the device
// (a9; K10 in §2.4).  All counting is integer and exact; means are formed on the host
// as (double)int64_sum / (double)count, so the result is bit-identical to the oracle.
//   f0-2   n_row, n_col, density
//   f3-5   nnz-per-row                  min/mean/max over rows
//   f6-8   nnz-blocks-per-row           |blocks_i|, blocks of bw columns (reading A14)
//   f9-11  warp load                    WL_w = sum_{p mod nw = w} ceil(nnz_p/nt) (Tab.II)
//   f12-14 same-cache-lines             requests per B line over lines with >= 1 request; a request =
//                                       one nt-nnz chunk of a row touching the line (A12)
//   f15-17 distinct-cache-lines-per-warp |union of blocks of rows p = w mod nw|
//   f18-20 total-cache-lines-per-warp   sum over the warp's rows and chunks of distinct lines per chunk
//   f21-23 adjacent-vector-distance     Hamming(mask_p, mask_{p+1}) (A13)
// "row p" is original row p (use_current_order = 0) or the row at position p of the current permutation.
#include "internal.cuh"
#include <algorithm>
#include <climits>
#include <vector>

namespace spmm {
namespace {

struct Stats {
    unsigned long long mn, mx, sum, cnt;
};

__device__ __forceinline__ void stats_add(Stats *st, long long v) {
    atomicMin(&st->mn, (unsigned long long)v);
    atomicMax(&st->mx, (unsigned long long)v);
    atomicAdd(&st->sum, (unsigned long long)v);
    atomicAdd(&st->cnt, 1ULL);
}

// warp-aggregated stats of non-negative values
__device__ __forceinline__ void warp_stats(Stats *st, long long v, bool valid) {
    unsigned long long mn = valid ? (unsigned long long)v : ~0ULL, mx = valid ? (unsigned long long)v : 0ULL;
    unsigned long long sm = valid ? (unsigned long long)v : 0ULL, c = valid ? 1ULL : 0ULL;
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        sm += __shfl_xor_sync(0xffffffffu, sm, o);
        c += __shfl_xor_sync(0xffffffffu, c, o);
    }
    if ((threadIdx.x & 31) == 0 && c) {
        atomicMin(&st->mn, mn);
        atomicMax(&st->mx, mx);
        atomicAdd(&st->sum, sm);
        atomicAdd(&st->cnt, c);
    }
}

// access to "row p": (start, end) and column j of the chosen CSR
struct OrigCSR {
    const int32_t *rowidx, *colidx, *perm;   // perm == nullptr: identity
    __device__ int32_t row(int64_t p) const { return perm ? perm[p] : (int32_t)p; }
    __device__ int32_t begin(int64_t p) const { return rowidx[row(p)]; }
    __device__ int32_t end(int64_t p) const { return rowidx[row(p) + 1]; }
    __device__ int32_t col(int32_t j) const { return colidx[j]; }
};

// per row p (warp): nnz, distinct blocks, warp load into WL[p % nw], distinct lines per nt-chunk
// (requests per line and T[p % nw]), union bitmap per warp-class (D), all exact integers.
__global__ void k_feat_rows(OrigCSR A, int64_t M, int32_t nw, int32_t nt, int32_t bw, int64_t words, Stats *st_nnz,
                            Stats *st_blk, unsigned long long *WL, unsigned long long *T, unsigned int *req,
                            uint32_t *Dmap, int32_t *nblk_row) {
    const int lane = threadIdx.x & 31;
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw_total = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t p0 = wid * 32; p0 < M; p0 += nw_total * 32) {
        // 32 rows per warp iteration; per-row stats aggregated across lanes first
        int32_t my_nnz = 0, my_blk = 0;
        bool my_valid = false;
        for (int r = 0; r < 32; ++r) {
            const int64_t p = p0 + r;
            if (p >= M) break;
            const int32_t a = A.begin(p), b = A.end(p);
            const int w = (int)(p % nw);
            int32_t blocks = 0, lines = 0;
            for (int32_t j0 = a; j0 < b; j0 += 32) {
                const int32_t j = j0 + lane;
                const bool in = j < b;
                const int32_t blk = in ? A.col(j) / bw : -1;
                const int32_t prv = (in && j > a) ? A.col(j - 1) / bw : -2;
                const bool newblk = in && (j == a || blk != prv);
                // chunk boundary: chunk = (j - a) / nt; first nnz of a chunk always counts as a new line
                const bool chunk_first = in && ((j - a) % nt == 0);
                const bool newline = in && (chunk_first || blk != prv);
                blocks += __popc(__ballot_sync(0xffffffffu, newblk));
                lines += __popc(__ballot_sync(0xffffffffu, newline));
                if (newline) atomicAdd(&req[blk], 1u);
                if (newblk) atomicOr(&Dmap[(size_t)w * words + (blk >> 5)], 1u << (blk & 31));
            }
            if (lane == 0) {
                atomicAdd(&WL[w], (unsigned long long)((b - a + nt - 1) / nt));
                atomicAdd(&T[w], (unsigned long long)lines);
                nblk_row[p] = blocks;
            }
            if (lane == r) { my_nnz = b - a; my_blk = blocks; my_valid = true; }
        }
        warp_stats(st_nnz, my_nnz, my_valid);
        warp_stats(st_blk, my_blk, my_valid);
    }
}

// stats over an unsigned array (skip zeros when requested)
__global__ void k_stats_u32(const unsigned int *v, int64_t n, int skip_zero, Stats *st) {
    for (int64_t i0 = (int64_t)blockIdx.x * blockDim.x; i0 < n; i0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = i0 + threadIdx.x;
        const bool in = i < n;
        const unsigned int x = in ? v[i] : 0u;
        warp_stats(st, x, in && (!skip_zero || x > 0));
    }
}

__global__ void k_popcount_rows(const uint32_t *Dmap, int64_t words, unsigned long long *D) {
    // one block per warp-class w
    unsigned long long c = 0;
    for (int64_t t = threadIdx.x; t < words; t += blockDim.x) c += __popc(Dmap[(size_t)blockIdx.x * words + t]);
#pragma unroll
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(&D[blockIdx.x], c);
}

// adjacent-vector distance: Hamming(p, p+1) = |b_p| + |b_{p+1}| - 2|common|.  Pairs whose rows hold at most
// ADJ_SHORT nnz together: thread per pair, merge of the two sorted (non-decreasing, duplicated) block sequences.
// Longer pairs (power-law hub rows, up to 10^5 nnz): warp per pair -- the lanes take the distinct blocks of the
// shorter row (run starts) and binary-search each in the longer row's columns -- so no single thread walks a hub row.
constexpr int32_t ADJ_SHORT = 256;
constexpr int32_t ADJ_HUGE = 2048;   // both rows longer: the pair goes to k_adjacent_huge (a CTA per pair)
__device__ __forceinline__ int32_t adj_common_merge(const OrigCSR &A, int64_t p, int32_t bw) {
    int32_t i = A.begin(p), ie = A.end(p), j = A.begin(p + 1), je = A.end(p + 1);
    int32_t common = 0;
    while (i < ie && j < je) {
        const int32_t x = A.col(i) / bw, y = A.col(j) / bw;
        if (x == y) {
            ++common;
            while (i < ie && A.col(i) / bw == x) ++i;
            while (j < je && A.col(j) / bw == y) ++j;
        } else if (x < y) {
            ++i;
        } else {
            ++j;
        }
    }
    return common;
}
__global__ void k_adjacent(OrigCSR A, int64_t M, int32_t bw, const int32_t *nblk_row, Stats *st, int64_t *huge,
                           unsigned long long *n_huge) {
    const int lane = threadIdx.x & 31;
    for (int64_t p0 = (int64_t)blockIdx.x * blockDim.x; p0 < M - 1; p0 += (int64_t)gridDim.x * blockDim.x) {
        const int64_t p = p0 + threadIdx.x;
        long long hd = 0;
        const bool in = p < M - 1;
        bool lng = false;
        int32_t b0 = 0, e0 = 0, b1 = 0, e1 = 0;
        if (in) {
            b0 = A.begin(p); e0 = A.end(p); b1 = A.begin(p + 1); e1 = A.end(p + 1);
            lng = (e0 - b0) + (e1 - b1) > ADJ_SHORT;
            if (!lng) hd = (long long)nblk_row[p] + nblk_row[p + 1] - 2LL * adj_common_merge(A, p, bw);
        }
        // pairs of two hub rows: deferred to k_adjacent_huge (their statistic is added there)
        const bool hg = lng && min(e0 - b0, e1 - b1) > ADJ_HUGE;
        if (hg) huge[atomicAdd(n_huge, 1ULL)] = p;
        lng = lng && !hg;
        // the warp's long pairs, one after another, all lanes together
        unsigned todo = __ballot_sync(0xffffffffu, lng);
        while (todo) {
            const int src = __ffs(todo) - 1;
            todo &= todo - 1;
            const int32_t sb0 = __shfl_sync(0xffffffffu, b0, src), se0 = __shfl_sync(0xffffffffu, e0, src);
            const int32_t sb1 = __shfl_sync(0xffffffffu, b1, src), se1 = __shfl_sync(0xffffffffu, e1, src);
            const bool first_short = se0 - sb0 <= se1 - sb1;
            const int32_t sb = first_short ? sb0 : sb1, se = first_short ? se0 : se1;   // scanned row
            const int32_t tb = first_short ? sb1 : sb0, te = first_short ? se1 : se0;   // searched row
            int32_t c = 0;
            for (int32_t i = sb + lane; i < se; i += 32) {
                const int32_t x = A.col(i) / bw;
                if (i > sb && A.col(i - 1) / bw == x) continue;   // not the first column of its block
                int32_t lo = tb, hi = te;                           // first column with block >= x
                while (lo < hi) {
                    const int32_t mid = (lo + hi) >> 1;
                    if (A.col(mid) / bw < x) lo = mid + 1;
                    else hi = mid;
                }
                c += lo < te && A.col(lo) / bw == x;
            }
#pragma unroll
            for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
            if (lane == src) hd = (long long)nblk_row[p] + nblk_row[p + 1] - 2LL * c;
        }
        warp_stats(st, hd, in && !hg);
    }
}

// the deferred pairs of two rows above ADJ_HUGE nnz: a CTA per pair, its threads take the shorter row's distinct
// blocks and binary-search them in the longer row
__global__ void k_adjacent_huge(OrigCSR A, int32_t bw, const int32_t *nblk_row, const int64_t *huge,
                                const unsigned long long *n_huge, Stats *st) {
    __shared__ int32_t part[32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (unsigned long long k = blockIdx.x; k < *n_huge; k += gridDim.x) {
        const int64_t p = huge[k];
        const int32_t b0 = A.begin(p), e0 = A.end(p), b1 = A.begin(p + 1), e1 = A.end(p + 1);
        const bool first_short = e0 - b0 <= e1 - b1;
        const int32_t sb = first_short ? b0 : b1, se = first_short ? e0 : e1;
        const int32_t tb = first_short ? b1 : b0, te = first_short ? e1 : e0;
        int32_t c = 0;
        for (int32_t i = sb + (int32_t)threadIdx.x; i < se; i += blockDim.x) {
            const int32_t x = A.col(i) / bw;
            if (i > sb && A.col(i - 1) / bw == x) continue;
            int32_t lo = tb, hi = te;
            while (lo < hi) {
                const int32_t mid = (lo + hi) >> 1;
                if (A.col(mid) / bw < x) lo = mid + 1;
                else hi = mid;
            }
            c += lo < te && A.col(lo) / bw == x;
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
        if (lane == 0) part[wid] = c;
        __syncthreads();
        if (threadIdx.x == 0) {
            int32_t t = 0;
            for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += part[w];
            stats_add(st, (long long)nblk_row[p] + nblk_row[p + 1] - 2LL * t);
        }
        __syncthreads();
    }
}

void put3(double *out, const Stats &s, bool empty_zero = true) {
    if (s.cnt == 0 && empty_zero) { out[0] = out[1] = out[2] = 0.0; return; }
    out[0] = (double)(long long)s.mn;
    out[1] = (double)(long long)s.sum / (double)(long long)s.cnt;
    out[2] = (double)(long long)s.mx;
}

void put3_vec(double *out, const std::vector<unsigned long long> &v) {
    if (v.empty()) { out[0] = out[1] = out[2] = 0.0; return; }
    unsigned long long mn = v[0], mx = v[0], sm = 0;
    for (auto x : v) { mn = std::min(mn, x); mx = std::max(mx, x); sm += x; }
    out[0] = (double)(long long)mn;
    out[1] = (double)(long long)sm / (double)v.size();
    out[2] = (double)(long long)mx;
}

}  // namespace

spmm_status compute_features(spmm_ctx *h, bool current_order, const spmm_params &p, double out[24], cudaStream_t s) {
    const int64_t M = h->M, N = h->N, nnz = h->nnz;
    const int32_t nw = p.nw, nt = p.nt, bw = p.bw;
    out[0] = (double)M;
    out[1] = (double)N;
    out[2] = (M && N) ? (double)nnz / ((double)M * (double)N) : 0.0;
    for (int i = 3; i < 24; ++i) out[i] = 0.0;
    if (M == 0) return SPMM_OK;
    const int64_t nblk = ceil_div(N, bw);
    const int64_t words = std::max<int64_t>(1, ceil_div(nblk, 32));
    DevBuf st, wl, tt, dd, req, dmap, nbr;
    SPMM_TRY(st.alloc(4 * sizeof(Stats), s));
    SPMM_TRY(wl.alloc(nw * sizeof(unsigned long long), s));
    SPMM_TRY(tt.alloc(nw * sizeof(unsigned long long), s));
    SPMM_TRY(dd.alloc(nw * sizeof(unsigned long long), s));
    SPMM_TRY(req.alloc(std::max<int64_t>(nblk, 1) * sizeof(unsigned int), s));
    SPMM_TRY(dmap.alloc((size_t)nw * words * sizeof(uint32_t), s));
    SPMM_TRY(nbr.alloc(M * sizeof(int32_t), s));
    Stats init[4];
    for (auto &x : init) { x.mn = ~0ULL; x.mx = 0; x.sum = 0; x.cnt = 0; }
    SPMM_CUDA(cudaMemcpyAsync(st.p, init, sizeof(init), cudaMemcpyHostToDevice, s));
    SPMM_CUDA(cudaMemsetAsync(wl.p, 0, wl.bytes, s));
    SPMM_CUDA(cudaMemsetAsync(tt.p, 0, tt.bytes, s));
    SPMM_CUDA(cudaMemsetAsync(dd.p, 0, dd.bytes, s));
    SPMM_CUDA(cudaMemsetAsync(req.p, 0, req.bytes, s));
    SPMM_CUDA(cudaMemsetAsync(dmap.p, 0, dmap.bytes, s));
    OrigCSR A{h->rowidx.as<int32_t>(), h->colidx.as<int32_t>(), current_order ? h->perm.as<int32_t>() : nullptr};
    Stats *S = st.as<Stats>();   // 0 nnz/row, 1 blocks/row, 2 requests, 3 adjacent
    const unsigned gw = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(M, 32 * 8), 148 * 16));
    k_feat_rows<<<gw, 256, 0, s>>>(A, M, nw, nt, bw, words, S + 0, S + 1, wl.as<unsigned long long>(),
                                   tt.as<unsigned long long>(), req.as<unsigned int>(), dmap.as<uint32_t>(),
                                   nbr.as<int32_t>());
    SPMM_CUDA(cudaGetLastError());
    k_stats_u32<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(nblk, 256), 148 * 16)), 256, 0, s>>>(
        req.as<unsigned int>(), nblk, 1, S + 2);
    k_popcount_rows<<<nw, 256, 0, s>>>(dmap.as<uint32_t>(), words, dd.as<unsigned long long>());
    DevBuf huge;
    if (M > 1) {
        // room for every pair whose rows both exceed ADJ_HUGE nnz (at most nnz / ADJ_HUGE of them) + the counter
        const int64_t cap = h->nnz / ADJ_HUGE + 2;
        SPMM_TRY(huge.alloc((size_t)(cap + 1) * sizeof(int64_t), s));
        unsigned long long *n_huge = reinterpret_cast<unsigned long long *>(huge.as<int64_t>() + cap);
        SPMM_CUDA(cudaMemsetAsync(n_huge, 0, sizeof(unsigned long long), s));
        k_adjacent<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(M, 256), 148 * 16)), 256, 0, s>>>(
            A, M, bw, nbr.as<int32_t>(), S + 3, huge.as<int64_t>(), n_huge);
        k_adjacent_huge<<<148 * 4, 256, 0, s>>>(A, bw, nbr.as<int32_t>(), huge.as<int64_t>(), n_huge, S + 3);
    }
    SPMM_CUDA(cudaGetLastError());
    Stats hs[4];
    std::vector<unsigned long long> hwl(nw), htt(nw), hdd(nw);
    SPMM_CUDA(cudaMemcpyAsync(hs, st.p, sizeof(hs), cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaMemcpyAsync(hwl.data(), wl.p, wl.bytes, cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaMemcpyAsync(htt.data(), tt.p, tt.bytes, cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaMemcpyAsync(hdd.data(), dd.p, dd.bytes, cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    put3(out + 3, hs[0]);
    put3(out + 6, hs[1]);
    put3_vec(out + 9, hwl);
    put3(out + 12, hs[2]);
    put3_vec(out + 15, hdd);
    put3_vec(out + 18, htt);
    put3(out + 21, hs[3]);
    return SPMM_OK;
}

// ---- B200 platform features g0..g6 (readings A24-A26) ------------------------
//   g0/g1  union of the columns of R = 2 / 4 consecutive positions, summed, per nnz (row fusion's B loads per nnz)
//   g2     distinct columns per window of 1024 consecutive positions, summed, per nnz
//   g3     4K*Cn / (4(M+1) + 8nnz + 4K*Cn + 4MK), Cn = distinct columns with >= 1 nnz
//   g4     empty positions / M;  g5  nnz in rows longer than 128 / nnz
//   g6     lane-slot efficiency of the short rows (0 < len <= 128): windows of 32 in position order, lengths
//          sorted descending, RPW at a time (8 if K <= 32, 4 if K <= 256, else 2): sum len / sum RPW * group max
// Integer counting on the device; the ratios are formed on the host as (double)int64 / (double)int64.
namespace {

enum { B_U2 = 0, B_U4, B_WIN, B_CN, B_EMPTY, B_SPLIT, B_SSUM, B_SLOTS, B_NCNT };

__device__ __forceinline__ void warp_add(unsigned long long *dst, unsigned long long v) {
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(dst, v);
}

// thread per group of R consecutive positions: R-way merge of the (strictly increasing) column lists
template <int R>
__global__ void k_b200_union(OrigCSR A, int64_t M, unsigned long long *out) {
    const int64_t ng = (M + R - 1) / R;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t g0 = (int64_t)blockIdx.x * blockDim.x; g0 < ng; g0 += stride) {
        const int64_t g = g0 + threadIdx.x;
        unsigned long long n = 0;
        if (g < ng) {
            int32_t j[R], e[R], c[R];
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int64_t p = g * R + r;
                j[r] = p < M ? A.begin(p) : 0;
                e[r] = p < M ? A.end(p) : 0;
                c[r] = j[r] < e[r] ? A.col(j[r]) : INT_MAX;
            }
            for (;;) {
                int32_t m = c[0];
#pragma unroll
                for (int r = 1; r < R; ++r) m = min(m, c[r]);
                if (m == INT_MAX) break;
#pragma unroll
                for (int r = 0; r < R; ++r)
                    if (c[r] == m) { ++j[r]; c[r] = j[r] < e[r] ? A.col(j[r]) : INT_MAX; }
                ++n;
            }
        }
        warp_add(out, n);
    }
}

__global__ void k_b200_rows(OrigCSR A, int64_t M, int32_t *len, int32_t *is_short, unsigned long long *out) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t p0 = (int64_t)blockIdx.x * blockDim.x; p0 < M; p0 += stride) {
        const int64_t p = p0 + threadIdx.x;
        int32_t l = 0;
        if (p < M) {
            l = A.end(p) - A.begin(p);
            len[p] = l;
            is_short[p] = l > 0 && l <= 128;
        }
        warp_add(out + B_EMPTY, (p < M && l == 0) ? 1ULL : 0ULL);
        warp_add(out + B_SPLIT, l > 128 ? (unsigned long long)l : 0ULL);
    }
}

// keys (window << 32 | col) of every nnz in position order (warp per position)
__global__ void k_b200_winkeys(OrigCSR A, int64_t M, const int32_t *pos_off, uint64_t *keys, uint32_t *vals) {
    const int lane = threadIdx.x & 31;
    for (int64_t p = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; p < M;
         p += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int32_t a = A.begin(p), l = A.end(p) - a, o = pos_off[p];
        const uint64_t w = (uint64_t)(p >> 10) << 32;
        for (int32_t t = lane; t < l; t += 32) {
            keys[o + t] = w | (uint32_t)A.col(a + t);
            vals[o + t] = 0u;
        }
    }
}

__global__ void k_b200_distinct(const uint64_t *keys, int64_t n, unsigned long long *out) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t j0 = (int64_t)blockIdx.x * blockDim.x; j0 < n; j0 += stride) {
        const int64_t j = j0 + threadIdx.x;
        warp_add(out, (j < n && (j == 0 || keys[j] != keys[j - 1])) ? 1ULL : 0ULL);
    }
}

__global__ void k_b200_colflags(const int32_t *colidx, int64_t nnz, uint8_t *flag) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nnz; j += (int64_t)gridDim.x * blockDim.x)
        flag[colidx[j]] = 1;
}

__global__ void k_b200_count_flags(const uint8_t *flag, int64_t n, unsigned long long *out) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t j0 = (int64_t)blockIdx.x * blockDim.x; j0 < n; j0 += stride) {
        const int64_t j = j0 + threadIdx.x;
        warp_add(out, (j < n && flag[j]) ? 1ULL : 0ULL);
    }
}

__global__ void k_b200_scatter_short(const int32_t *is_short, const int32_t *sidx, const int32_t *len, int64_t M,
                                     int32_t *slen) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < M; p += (int64_t)gridDim.x * blockDim.x)
        if (is_short[p]) slen[sidx[p]] = len[p];
}

// thread per window of 32 short rows: insertion sort descending, then RPW-groups
__global__ void k_b200_slots(const int32_t *slen, int64_t ns, int32_t rpw, unsigned long long *out) {
    const int64_t nwin = (ns + 31) / 32;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t w0 = (int64_t)blockIdx.x * blockDim.x; w0 < nwin; w0 += stride) {
        const int64_t w = w0 + threadIdx.x;
        unsigned long long sum = 0, slots = 0;
        if (w < nwin) {
            int32_t v[32];
            const int n = (int)(ns - w * 32 < 32 ? ns - w * 32 : 32);
            for (int t = 0; t < n; ++t) {
                int32_t x = slen[w * 32 + t];
                sum += (unsigned long long)x;
                int u = t;
                while (u > 0 && v[u - 1] < x) { v[u] = v[u - 1]; --u; }
                v[u] = x;
            }
            for (int t = 0; t < n; t += rpw) slots += (unsigned long long)rpw * (unsigned long long)v[t];
        }
        warp_add(out + B_SSUM, sum);
        warp_add(out + B_SLOTS, slots);
    }
}

inline unsigned gb(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 16)); }
inline double ratio(unsigned long long a, unsigned long long b) { return b ? (double)a / (double)b : 0.0; }

}  // namespace

spmm_status compute_features_b200(spmm_ctx *h, bool current_order, int64_t K, double out[7], cudaStream_t s) {
    const int64_t M = h->M, N = h->N, nnz = h->nnz;
    for (int i = 0; i < 7; ++i) out[i] = 0.0;
    if (M == 0) return SPMM_OK;
    OrigCSR A{h->rowidx.as<int32_t>(), h->colidx.as<int32_t>(), current_order ? h->perm.as<int32_t>() : nullptr};
    DevBuf cnt, len, is_short, sidx, slen, off, keys, vals, flag;
    SPMM_TRY(cnt.alloc(B_NCNT * sizeof(unsigned long long), s));
    SPMM_CUDA(cudaMemsetAsync(cnt.p, 0, cnt.bytes, s));
    unsigned long long *C = cnt.as<unsigned long long>();
    k_b200_union<2><<<gb(ceil_div(M, 2)), 256, 0, s>>>(A, M, C + B_U2);
    k_b200_union<4><<<gb(ceil_div(M, 4)), 256, 0, s>>>(A, M, C + B_U4);
    SPMM_TRY(len.alloc(M * sizeof(int32_t), s));
    SPMM_TRY(is_short.alloc(M * sizeof(int32_t), s));
    k_b200_rows<<<gb(M), 256, 0, s>>>(A, M, len.as<int32_t>(), is_short.as<int32_t>(), C);
    SPMM_CUDA(cudaGetLastError());
    if (nnz > 0) {
        // window distinct columns: sort (window, col) keys, count distinct
        SPMM_TRY(off.alloc((M + 1) * sizeof(int32_t), s));
        SPMM_TRY(exclusive_scan_i32(len.as<int32_t>(), off.as<int32_t>(), M, nullptr, s));
        SPMM_TRY(keys.alloc(nnz * sizeof(uint64_t), s));
        SPMM_TRY(vals.alloc(nnz * sizeof(uint32_t), s));
        k_b200_winkeys<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(M * 32, 256), 148 * 64)), 256, 0,
                         s>>>(A, M, off.as<int32_t>(), keys.as<uint64_t>(), vals.as<uint32_t>());
        SPMM_CUDA(cudaGetLastError());
        int hi = 32;
        while (hi < 64 && (((M - 1) >> 10) >> (hi - 32)) > 0) ++hi;
        SPMM_TRY(radix_sort_pairs(keys.as<uint64_t>(), vals.as<uint32_t>(), nnz, 0, ((hi + 7) / 8) * 8, s));
        k_b200_distinct<<<gb(nnz), 256, 0, s>>>(keys.as<uint64_t>(), nnz, C + B_WIN);
        keys.release();
        vals.release();
        // distinct columns overall
        SPMM_TRY(flag.alloc(std::max<int64_t>(N, 1), s));
        SPMM_CUDA(cudaMemsetAsync(flag.p, 0, flag.bytes, s));
        k_b200_colflags<<<gb(nnz), 256, 0, s>>>(h->colidx.as<int32_t>(), nnz, flag.as<uint8_t>());
        k_b200_count_flags<<<gb(N), 256, 0, s>>>(flag.as<uint8_t>(), N, C + B_CN);
        SPMM_CUDA(cudaGetLastError());
    }
    // lane-slot efficiency of the short rows
    SPMM_TRY(sidx.alloc((M + 1) * sizeof(int32_t), s));
    int32_t ns = 0;
    SPMM_TRY(exclusive_scan_i32(is_short.as<int32_t>(), sidx.as<int32_t>(), M, &ns, s));
    if (ns > 0) {
        SPMM_TRY(slen.alloc(ns * sizeof(int32_t), s));
        k_b200_scatter_short<<<gb(M), 256, 0, s>>>(is_short.as<int32_t>(), sidx.as<int32_t>(), len.as<int32_t>(), M,
                                                  slen.as<int32_t>());
        const int32_t rpw = K <= 32 ? 8 : K <= 256 ? 4 : 2;
        k_b200_slots<<<gb(ceil_div(ns, 32)), 256, 0, s>>>(slen.as<int32_t>(), ns, rpw, C);
        SPMM_CUDA(cudaGetLastError());
    }
    unsigned long long hc[B_NCNT];
    SPMM_CUDA(cudaMemcpyAsync(hc, cnt.p, sizeof(hc), cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    const unsigned long long nz = (unsigned long long)nnz;
    out[0] = ratio(hc[B_U2], nz);
    out[1] = ratio(hc[B_U4], nz);
    out[2] = ratio(hc[B_WIN], nz);
    const unsigned long long kb = 4ULL * (unsigned long long)K * hc[B_CN];
    out[3] = ratio(kb, 4ULL * (unsigned long long)(M + 1) + 8ULL * nz + kb + 4ULL * (unsigned long long)M * K);
    out[4] = ratio(hc[B_EMPTY], (unsigned long long)M);
    out[5] = ratio(hc[B_SPLIT], nz);
    out[6] = ratio(hc[B_SSUM], hc[B_SLOTS]);
    return SPMM_OK;
}

}  // namespace spmm
