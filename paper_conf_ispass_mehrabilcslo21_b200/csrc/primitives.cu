// primitives.cu -- device-wide scan, max-reduction and a stable LSD radix sort, hand-written for the
// permutation builders ("histogram -> exclusive scan -> stable scatter").
// These are HBM-bound helpers of spmm_permute (offline / amortised per P:L96), not the timed SpMM.
#include "internal.cuh"

namespace spmm {
namespace {

constexpr int SCAN_THREADS = 512;
constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;

template <class T>
__device__ T block_exclusive_scan(T v, T *smem_warp, T *total) {
    // v: this thread's value; returns exclusive prefix within the block; *total = block sum
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    T x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) smem_warp[wid] = x;
    __syncthreads();
    if (wid == 0) {
        constexpr int NW = SCAN_THREADS / 32;
        T w = lane < NW ? smem_warp[lane] : T(0);
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            T y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        if (lane < NW) smem_warp[lane] = w;   // inclusive warp totals
    }
    __syncthreads();
    T warp_off = wid ? smem_warp[wid - 1] : T(0);
    *total = smem_warp[SCAN_THREADS / 32 - 1];
    __syncthreads();
    return warp_off + x - v;
}

template <class T>
__global__ void __launch_bounds__(SCAN_THREADS) k_tile_sums(const T *in, int64_t n, T *sums) {
    __shared__ T sw[SCAN_THREADS / 32];
    int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
    T s = 0;
#pragma unroll
    for (int t = 0; t < SCAN_ITEMS; ++t)
        if (base + t < n) s += in[base + t];
    T tot;
    block_exclusive_scan<T>(s, sw, &tot);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

// exclusive scan of one tile with a tile offset; out has n+1 slots when write_total
template <class T>
__global__ void __launch_bounds__(SCAN_THREADS) k_tile_scan(const T *in, int64_t n, const T *offs, T *out,
                                                            int write_total) {
    __shared__ T sw[SCAN_THREADS / 32];
    int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
    T v[SCAN_ITEMS];
    T s = 0;
#pragma unroll
    for (int t = 0; t < SCAN_ITEMS; ++t) {
        v[t] = base + t < n ? in[base + t] : T(0);
        s += v[t];
    }
    T tot;
    T pre = block_exclusive_scan<T>(s, sw, &tot) + (offs ? offs[blockIdx.x] : T(0));
#pragma unroll
    for (int t = 0; t < SCAN_ITEMS; ++t) {
        if (base + t < n) out[base + t] = pre;
        pre += v[t];
    }
    if (write_total && base < n && base + SCAN_ITEMS >= n) out[n] = pre;   // the thread holding element n-1
}

template <class T>
spmm_status scan_impl(const T *in, T *out, int64_t n, int write_total, cudaStream_t s) {
    if (n == 0) {
        if (write_total) SPMM_CUDA(cudaMemsetAsync(out, 0, sizeof(T), s));
        return SPMM_OK;
    }
    int64_t tiles = ceil_div(n, SCAN_TILE);
    if (tiles == 1) {
        k_tile_scan<T><<<1, SCAN_THREADS, 0, s>>>(in, n, nullptr, out, write_total);
        SPMM_CUDA(cudaGetLastError());
        return SPMM_OK;
    }
    DevBuf sums, offs;
    SPMM_TRY(sums.alloc(tiles * sizeof(T), s));
    SPMM_TRY(offs.alloc(tiles * sizeof(T), s));
    k_tile_sums<T><<<(unsigned)tiles, SCAN_THREADS, 0, s>>>(in, n, sums.as<T>());
    SPMM_CUDA(cudaGetLastError());
    SPMM_TRY(scan_impl<T>(sums.as<T>(), offs.as<T>(), tiles, 0, s));
    k_tile_scan<T><<<(unsigned)tiles, SCAN_THREADS, 0, s>>>(in, n, offs.as<T>(), out, write_total);
    SPMM_CUDA(cudaGetLastError());
    return SPMM_OK;
}

__global__ void k_max_i32(const int32_t *in, int64_t n, int32_t *out) {
    int32_t m = INT32_MIN;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        m = max(m, in[i]);
#pragma unroll
    for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
    if ((threadIdx.x & 31) == 0) atomicMax(out, m);
}

// ---- stable LSD radix sort, 8-bit digits ---------------------------------------------------
constexpr int RS_THREADS = 256;
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_ROUNDS = 8;                         // 32-item rounds per warp
constexpr int RS_TILE = RS_THREADS * RS_ROUNDS;      // 2048 items per block

__global__ void __launch_bounds__(RS_THREADS) k_rs_hist(const uint64_t *keys, int64_t n, int shift,
                                                        int32_t *counts, int64_t nblocks) {
    __shared__ int32_t h[256];
    h[threadIdx.x] = 0;
    __syncthreads();
    int64_t base = (int64_t)blockIdx.x * RS_TILE;
    for (int t = threadIdx.x; t < RS_TILE; t += RS_THREADS) {
        int64_t i = base + t;
        if (i < n) atomicAdd(&h[(keys[i] >> shift) & 255u], 1);
    }
    __syncthreads();
    counts[(int64_t)threadIdx.x * nblocks + blockIdx.x] = h[threadIdx.x];   // digit-major
}

__global__ void __launch_bounds__(RS_THREADS) k_rs_scatter(const uint64_t *keys, const uint32_t *vals, int64_t n,
                                                           int shift, const int32_t *offsets, int64_t nblocks,
                                                           uint64_t *keys_out, uint32_t *vals_out) {
    __shared__ int32_t wc[RS_WARPS][256];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int d = lane; d < 256; d += 32) wc[wid][d] = 0;
    __syncwarp();
    const int64_t base = (int64_t)blockIdx.x * RS_TILE + (int64_t)wid * (32 * RS_ROUNDS);
    uint64_t k[RS_ROUNDS];
    uint32_t v[RS_ROUNDS];
    int32_t rank[RS_ROUNDS];
    uint32_t dig[RS_ROUNDS];
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int r = 0; r < RS_ROUNDS; ++r) {
        int64_t i = base + r * 32 + lane;
        bool ok = i < n;
        k[r] = ok ? keys[i] : 0;
        v[r] = ok ? vals[i] : 0;
        dig[r] = ok ? (uint32_t)((k[r] >> shift) & 255u) : 256u;
        unsigned peers = __match_any_sync(0xffffffffu, dig[r]);
        int leader = __ffs(peers) - 1;
        int prior = 0;
        if (ok) prior = wc[wid][dig[r]];
        rank[r] = prior + __popc(peers & lt);
        __syncwarp();
        if (ok && lane == leader) wc[wid][dig[r]] = prior + __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    // per digit: exclusive scan across warps, plus the block's global offset
    {
        int d = threadIdx.x;   // 256 threads == 256 digits
        int32_t run = offsets[(int64_t)d * nblocks + blockIdx.x];
#pragma unroll
        for (int w = 0; w < RS_WARPS; ++w) {
            int32_t c = wc[w][d];
            wc[w][d] = run;
            run += c;
        }
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < RS_ROUNDS; ++r) {
        if (dig[r] < 256u) {
            int32_t dst = wc[wid][dig[r]] + rank[r];
            keys_out[dst] = k[r];
            vals_out[dst] = v[r];
        }
    }
}

}  // namespace

spmm_status exclusive_scan_i32(const int32_t *in, int32_t *out, int64_t n, int32_t *total_host, cudaStream_t s) {
    SPMM_TRY(scan_impl<int32_t>(in, out, n, 1, s));
    if (total_host) {
        SPMM_CUDA(cudaMemcpyAsync(total_host, out + n, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
        SPMM_CUDA(cudaStreamSynchronize(s));
    }
    return SPMM_OK;
}

spmm_status exclusive_scan_i64(const int64_t *in, int64_t *out, int64_t n, cudaStream_t s) {
    return scan_impl<int64_t>(in, out, n, 1, s);
}

spmm_status reduce_max_i32(const int32_t *in, int64_t n, int32_t *result_host, cudaStream_t s) {
    DevBuf r;
    SPMM_TRY(r.alloc(sizeof(int32_t), s));
    int32_t init = INT32_MIN;
    SPMM_CUDA(cudaMemcpyAsync(r.p, &init, sizeof(init), cudaMemcpyHostToDevice, s));
    if (n > 0) {
        int blocks = (int)std::min<int64_t>(ceil_div(n, 256), 148 * 8);
        k_max_i32<<<blocks, 256, 0, s>>>(in, n, r.as<int32_t>());
        SPMM_CUDA(cudaGetLastError());
    }
    SPMM_CUDA(cudaMemcpyAsync(result_host, r.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    SPMM_CUDA(cudaStreamSynchronize(s));
    return SPMM_OK;
}

spmm_status radix_sort_pairs(uint64_t *keys, uint32_t *vals, int64_t n, int begin_bit, int end_bit, cudaStream_t s) {
    if (n <= 1 || end_bit <= begin_bit) return SPMM_OK;
    if (n >= ((int64_t)1 << 31)) return fail(SPMM_ERR_UNSUPPORTED, "radix sort: n >= 2^31");
    int64_t nblocks = ceil_div(n, RS_TILE);
    DevBuf k2, v2, counts, offsets;
    SPMM_TRY(k2.alloc(n * sizeof(uint64_t), s));
    SPMM_TRY(v2.alloc(n * sizeof(uint32_t), s));
    SPMM_TRY(counts.alloc(256 * nblocks * sizeof(int32_t), s));
    SPMM_TRY(offsets.alloc((256 * nblocks + 1) * sizeof(int32_t), s));
    uint64_t *kin = keys, *kout = k2.as<uint64_t>();
    uint32_t *vin = vals, *vout = v2.as<uint32_t>();
    int passes = 0;
    for (int shift = begin_bit; shift < end_bit; shift += 8, ++passes) {
        k_rs_hist<<<(unsigned)nblocks, RS_THREADS, 0, s>>>(kin, n, shift, counts.as<int32_t>(), nblocks);
        SPMM_CUDA(cudaGetLastError());
        SPMM_TRY(scan_impl<int32_t>(counts.as<int32_t>(), offsets.as<int32_t>(), 256 * nblocks, 0, s));
        k_rs_scatter<<<(unsigned)nblocks, RS_THREADS, 0, s>>>(kin, vin, n, shift, offsets.as<int32_t>(), nblocks,
                                                              kout, vout);
        SPMM_CUDA(cudaGetLastError());
        std::swap(kin, kout);
        std::swap(vin, vout);
    }
    if (passes & 1) {
        SPMM_CUDA(cudaMemcpyAsync(keys, kin, n * sizeof(uint64_t), cudaMemcpyDeviceToDevice, s));
        SPMM_CUDA(cudaMemcpyAsync(vals, vin, n * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
    }
    return SPMM_OK;
}

}  // namespace spmm
