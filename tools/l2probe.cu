// tools/l2probe.cu -- measurement helper (not the method): achievable L2->SM read bandwidth on this GPU.
// Every warp streams float4 loads over an L2-resident buffer (size < L2) `reps` times; the sum is
// written out so the loads are not dead.  Returns bytes/second via CUDA events.
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void __launch_bounds__(256) k_l2read(const float4 *__restrict__ buf, int64_t n4, int reps, float *out) {
    float acc = 0.f;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int r = 0; r < reps; ++r) {
        for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride * 4) {
            float4 a = __ldcg(buf + i);
            float4 b = i + stride < n4 ? __ldcg(buf + i + stride) : make_float4(0, 0, 0, 0);
            float4 c = i + 2 * stride < n4 ? __ldcg(buf + i + 2 * stride) : make_float4(0, 0, 0, 0);
            float4 d = i + 3 * stride < n4 ? __ldcg(buf + i + 3 * stride) : make_float4(0, 0, 0, 0);
            acc += a.x + a.y + a.z + a.w + b.x + b.y + b.z + b.w + c.x + c.y + c.z + c.w + d.x + d.y + d.z + d.w;
        }
    }
    out[(int64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

extern "C" double l2probe_read_bw(int64_t bytes, int reps) {
    int sms = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    float4 *buf = nullptr;
    float *out = nullptr;
    const int blocks = sms * 8, threads = 256;
    if (cudaMalloc(&buf, bytes) != cudaSuccess) return -1.0;
    cudaMalloc(&out, (size_t)blocks * threads * sizeof(float));
    cudaMemset(buf, 0, bytes);
    const int64_t n4 = bytes / 16;
    k_l2read<<<blocks, threads>>>(buf, n4, 2, out);   // warm L2
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    k_l2read<<<blocks, threads>>>(buf, n4, reps, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    cudaFree(buf);
    cudaFree(out);
    return (double)bytes * reps / (ms * 1e-3);
}

// Per-SM view: only CTAs resident on SMs with smid < limit read (each warp a private 32 KB slice of the
// L2-resident buffer, `reps` times); returns the aggregate bytes/second of those SMs.  Comparing limit =
// all SMs with limit = half tells whether the L2->SM ceiling is per-SM ingress or the L2 slices.
__global__ void __launch_bounds__(256) k_l2read_sms(const float4 *__restrict__ buf, int64_t n4, int reps, int limit,
                                                   unsigned long long *bytes, float *out) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    if ((int)smid >= limit) return;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    const int64_t slice = 2048;                     // float4 per warp = 32 KB
    const int64_t base = (warp * slice) % (n4 - slice);
    float acc = 0.f;
    for (int r = 0; r < reps; ++r)
        for (int64_t i = lane; i < slice; i += 128) {
            float4 a = __ldcg(buf + base + i), b = __ldcg(buf + base + i + 32), c = __ldcg(buf + base + i + 64),
                   d = __ldcg(buf + base + i + 96);
            acc += a.x + b.y + c.z + d.w;
        }
    out[(int64_t)blockIdx.x * blockDim.x + threadIdx.x] = acc;
    if (lane == 0) atomicAdd(bytes, (unsigned long long)(slice * 16 * reps));
}

extern "C" double l2probe_read_bw_sms(int64_t bytes_, int reps, int limit) {
    int sms = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    float4 *buf = nullptr;
    float *out = nullptr;
    unsigned long long *cnt = nullptr;
    const int blocks = sms * 8, threads = 256;
    if (cudaMalloc(&buf, bytes_) != cudaSuccess) return -1.0;
    cudaMalloc(&out, (size_t)blocks * threads * sizeof(float));
    cudaMalloc(&cnt, sizeof(unsigned long long));
    cudaMemset(buf, 0, bytes_);
    const int64_t n4 = bytes_ / 16;
    k_l2read_sms<<<blocks, threads>>>(buf, n4, 1, sms, cnt, out);   // warm
    cudaMemset(cnt, 0, sizeof(unsigned long long));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    k_l2read_sms<<<blocks, threads>>>(buf, n4, reps, limit, cnt, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    unsigned long long b = 0;
    cudaMemcpy(&b, cnt, sizeof(b), cudaMemcpyDeviceToHost);
    cudaFree(buf);
    cudaFree(out);
    cudaFree(cnt);
    return (double)b / (ms * 1e-3);
}
