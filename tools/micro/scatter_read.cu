// Microbenchmark: DRAM bytes fetched per scattered 4-byte read (one word per
// 6400-byte row, 1.44 M rows: the x-wall nodes of the C4 hall) for several
// load flavours, and with cudaLimitMaxL2FetchGranularity.  Run under ncu with
// dram__bytes_read.sum.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 scatter_read.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int V>
__global__ void rd(const float *a, float *out, long n, long stride)
{
    long i = blockIdx.x * (long)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const float *p = a + i * stride;
    float v;
    if (V == 0) v = *p;
    if (V == 1) asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(v) : "l"(p));
    if (V == 2) asm volatile("ld.global.cs.f32 %0, [%1];" : "=f"(v) : "l"(p));
    if (V == 3) asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(v) : "l"(p));
    if (V == 4) asm volatile("ld.global.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    if (V == 5) asm volatile("ld.relaxed.gpu.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
    if (V == 6) asm volatile("ld.volatile.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
    if (V == 7) {  // evict_first policy
        uint64_t pol;
        asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
        asm volatile("ld.global.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    }
    if (v == 12345.f) out[0] = 1.f;
}
__global__ void flush(float *b, long n)
{
    long i = blockIdx.x * (long)blockDim.x + threadIdx.x;
    if (i < n) b[i] = b[i] + 1.0f;
}

int main()
{
    const long stride = 1600, n = 1441792;
    float *a, *b, *o;
    cudaMalloc(&a, n * stride * 4 + 64);
    cudaMalloc(&b, 512l << 20);
    cudaMalloc(&o, 64);
    cudaMemset(a, 0, n * stride * 4);
    const long fb = (512l << 20) / 4;
    const int gran[] = {-1, 32, 64, 128};
    for (int gi = 0; gi < 4; gi++) {
        if (gran[gi] > 0) {
            cudaError_t e = cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, gran[gi]);
            size_t got = 0;
            cudaDeviceGetLimit(&got, cudaLimitMaxL2FetchGranularity);
            printf("granularity %d: %s (now %zu)\n", gran[gi], cudaGetErrorString(e), got);
        }
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        for (int v = 0; v < 8; v++) {
            flush<<<(fb + 255) / 256, 256>>>(b, fb);
            cudaEventRecord(e0);
            const unsigned g = (unsigned)((n + 255) / 256);
            switch (v) {
                case 0: rd<0><<<g, 256>>>(a, o, n, stride); break;
                case 1: rd<1><<<g, 256>>>(a, o, n, stride); break;
                case 2: rd<2><<<g, 256>>>(a, o, n, stride); break;
                case 3: rd<3><<<g, 256>>>(a, o, n, stride); break;
                case 4: rd<4><<<g, 256>>>(a, o, n, stride); break;
                case 5: rd<5><<<g, 256>>>(a, o, n, stride); break;
                case 6: rd<6><<<g, 256>>>(a, o, n, stride); break;
                case 7: rd<7><<<g, 256>>>(a, o, n, stride); break;
            }
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            printf("gran %d variant %d: %.1f us\n", gran[gi], v, ms * 1e3);
        }
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
