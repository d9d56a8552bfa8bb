// Streaming bandwidth of k_volume2's traffic mix without its access pattern:
// per element read two fp32 arrays and one byte array, write two fp32 arrays
// (17 bytes, 53 % reads by bytes ... as one double step of the two-step sweep),
// plus a plain copy (the MEASURED_PEAKS.json recipe: read + write) and the
// single-step mix (read 2 x fp32 + 1 byte, write 1 x fp32: 13 bytes).
// 16-byte vector accesses, grid-stride, CUDA events, best of 10.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 stream_mix.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void mix2(const float4 *a, const float4 *b, const uint32_t *k, float4 *d, float4 *e, long n4)
{
    for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n4; i += (long)gridDim.x * blockDim.x) {
        float4 x = a[i], y = b[i];
        uint32_t kk = k[i];
        float f = (float)(kk & 7);
        d[i] = make_float4(x.x + y.x, x.y + y.y, x.z + y.z, x.w + f);
        e[i] = make_float4(x.x - y.x, x.y - y.y, x.z - y.z, x.w - f);
    }
}
__global__ void mix1(const float4 *a, const float4 *b, const uint32_t *k, float4 *d, long n4)
{
    for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n4; i += (long)gridDim.x * blockDim.x) {
        float4 x = a[i], y = b[i];
        float f = (float)(k[i] & 7);
        d[i] = make_float4(x.x + y.x, x.y + y.y, x.z + y.z, x.w + f);
    }
}
__global__ void copy(const float4 *a, float4 *d, long n4)
{
    for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n4; i += (long)gridDim.x * blockDim.x) d[i] = a[i];
}

int main()
{
    const long n = 1107296256l;  // the C4 hall's voxels
    const long n4 = n / 4;
    float4 *a, *b, *d, *e;
    uint32_t *k;
    cudaMalloc(&a, n * 4);
    cudaMalloc(&b, n * 4);
    cudaMalloc(&d, n * 4);
    cudaMalloc(&e, n * 4);
    cudaMalloc(&k, n);
    cudaMemset(a, 0, n * 4);
    cudaMemset(b, 0, n * 4);
    cudaMemset(k, 6, n);
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int v = 0; v < 3; v++) {
        for (int bpsm = 4; bpsm <= 16; bpsm *= 2) {
            float best = 1e30f;
            for (int rep = 0; rep < 10; rep++) {
                cudaEventRecord(e0);
                if (v == 0) mix2<<<nsm * bpsm, 256>>>(a, b, k, d, e, n4);
                if (v == 1) mix1<<<nsm * bpsm, 256>>>(a, b, k, d, n4);
                if (v == 2) copy<<<nsm * bpsm, 256>>>(a, d, n4);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                if (ms < best) best = ms;
            }
            const double bytes = v == 0 ? 17.0 * n : v == 1 ? 13.0 * n : 8.0 * n;
            const char *nm[] = {"two-step mix (R 4+4+1, W 4+4 B)", "single-step mix (R 4+4+1, W 4 B)", "copy (R 4, W 4 B)"};
            printf("%-34s blocks/SM %2d: %.3f ms  %.1f GB/s\n", nm[v], bpsm, best, bytes / (best * 1e-3) / 1e9);
        }
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
