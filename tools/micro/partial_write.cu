// Microbenchmark: DRAM cost of scattered partial-sector writes vs full-sector
// writes vs scattered 4-byte reads (one 4-byte word per 6400-byte row, like the
// x-wall nodes of the C4 hall).  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 partial_write.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void w4(float *a, long n, long stride)  // 4 B into each row's first sector
{
    long i = blockIdx.x * (long)blockDim.x + threadIdx.x;
    if (i < n) a[i * stride] = 1.0f;
}
__global__ void w32(float *a, long n, long stride)  // the row's whole first sector (8 lanes per row)
{
    long t = blockIdx.x * (long)blockDim.x + threadIdx.x;
    long i = t >> 3;
    if (i < n) a[i * stride + (t & 7)] = 1.0f;
}
__global__ void r4(const float *a, float *out, long n, long stride)
{
    long i = blockIdx.x * (long)blockDim.x + threadIdx.x;
    if (i < n && a[i * stride] == 12345.f) out[0] = 1.f;
}
__global__ void rw4(float *a, long n, long stride)  // read-modify-write of one word
{
    long i = blockIdx.x * (long)blockDim.x + threadIdx.x;
    if (i < n) a[i * stride] = a[i * stride] * 0.5f + 1.0f;
}
__global__ void flush(float *b, long n)
{
    long i = blockIdx.x * (long)blockDim.x + threadIdx.x;
    if (i < n) b[i] = b[i] + 1.0f;
}

int main()
{
    const long stride = 1600;     // floats per row (C4 pitch)
    const long n = 1441792;       // rows (1024 x 1408: the C4 x-wall count)
    float *a, *b, *o;
    cudaMalloc(&a, n * stride * 4 + 64);
    cudaMalloc(&b, 512l << 20);
    cudaMalloc(&o, 64);
    cudaMemset(a, 0, n * stride * 4);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const long fb = (512l << 20) / 4;
    for (int rep = 0; rep < 3; rep++) {
        for (int k = 0; k < 4; k++) {
            flush<<<(fb + 255) / 256, 256>>>(b, fb);
            cudaEventRecord(e0);
            if (k == 0) w4<<<(n + 255) / 256, 256>>>(a, n, stride);
            if (k == 1) w32<<<(n * 8 + 255) / 256, 256>>>(a, n, stride);
            if (k == 2) r4<<<(n + 255) / 256, 256>>>(a, o, n, stride);
            if (k == 3) rw4<<<(n + 255) / 256, 256>>>(a, n, stride);
            cudaEventRecord(e1);
            flush<<<(fb + 255) / 256, 256>>>(b, fb);  // pushes dirty lines out (write-back inside this kernel)
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            const char *nm[] = {"write 4 B / row", "write 32 B / row", "read 4 B / row", "read+write 4 B / row"};
            printf("%-22s %8.1f us\n", nm[k], ms * 1e3);
        }
    }
    cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
