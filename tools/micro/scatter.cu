// Micro-benchmark: random 4/8-byte gathers vs scatters vs atomics on B200.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scatter scatter.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <vector>
#include <algorithm>
#include <random>

__global__ void k_gather(const uint32_t *perm, const uint2 *src, uint2 *dst, int n) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        dst[i] = src[perm[i]];
}
template <int ILP>
__global__ void k_scatter(const uint32_t *perm, const uint2 *src, uint2 *dst, int n) {
    const int stride = gridDim.x * blockDim.x;
    for (int i0 = blockIdx.x * blockDim.x + threadIdx.x; i0 < n; i0 += stride * ILP) {
        uint32_t p[ILP]; uint2 v[ILP];
#pragma unroll
        for (int k = 0; k < ILP; k++) { int i = i0 + k * stride; if (i < n) { p[k] = perm[i]; v[k] = src[i]; } }
#pragma unroll
        for (int k = 0; k < ILP; k++) { int i = i0 + k * stride; if (i < n) dst[p[k]] = v[k]; }
    }
}
__global__ void k_scatter4(const uint32_t *perm, uint32_t *dst, int n) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        dst[perm[i]] = i;
}
__global__ void k_atomic(const uint32_t *perm, uint32_t *dst, int n, int mod) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        atomicAdd(dst + perm[i] % mod, 1u);
}
__global__ void k_atomic_ret(const uint32_t *perm, uint32_t *dst, uint32_t *out, int n, int mod) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        out[i] = atomicAdd(dst + perm[i] % mod, 1u);
}
__global__ void k_copy(const uint2 *src, uint2 *dst, int n) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) dst[i] = src[i];
}

int main() {
    const int n = 10000000;
    std::vector<uint32_t> h(n);
    for (int i = 0; i < n; i++) h[i] = i;
    std::mt19937 rng(1);
    std::shuffle(h.begin(), h.end(), rng);
    uint32_t *perm, *d4, *o4; uint2 *src, *dst;
    cudaMalloc(&perm, 4ull * n); cudaMalloc(&src, 8ull * n); cudaMalloc(&dst, 8ull * n);
    cudaMalloc(&d4, 4ull * n); cudaMalloc(&o4, 4ull * n);
    cudaMemcpy(perm, h.data(), 4ull * n, cudaMemcpyHostToDevice);
    cudaMemset(src, 1, 8ull * n);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto T = [&](const char *name, auto fn) {
        for (int w = 0; w < 3; w++) fn();
        cudaEventRecord(a);
        for (int r = 0; r < 10; r++) fn();
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        printf("%-28s %8.1f us  %6.1f G/s\n", name, 100 * ms, n / (ms / 10 * 1e-3) / 1e9);
    };
    int g = sms * 8;
    T("copy 8B", [&] { k_copy<<<g, 256>>>(src, dst, n); });
    T("gather 8B (80MB src)", [&] { k_gather<<<g, 256>>>(perm, src, dst, n); });
    T("scatter 8B ilp1", [&] { k_scatter<1><<<g, 256>>>(perm, src, dst, n); });
    T("scatter 8B ilp4", [&] { k_scatter<4><<<g, 256>>>(perm, src, dst, n); });
    T("scatter 4B", [&] { k_scatter4<<<g, 256>>>(perm, d4, n); });
    T("atomic 4B no-ret (40MB)", [&] { k_atomic<<<g, 256>>>(perm, d4, n, n); });
    T("atomic 4B ret (40MB)", [&] { k_atomic_ret<<<g, 256>>>(perm, d4, o4, n, n); });
    T("atomic 4B ret (4MB)", [&] { k_atomic_ret<<<g, 256>>>(perm, d4, o4, n, 1000000); });
    T("atomic 4B no-ret (4MB)", [&] { k_atomic<<<g, 256>>>(perm, d4, n, 1000000); });
    cudaError_t e = cudaGetLastError();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
