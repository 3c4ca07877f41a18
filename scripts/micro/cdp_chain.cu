// Micro-benchmark: device-side launch chains (CDP2) on B200.
//  (a) tail-launch chain: k<<<g,b>>> tail-launches itself N times
//  (b) driver pattern: driver launches work (fire-and-forget) + tail-launches itself
//  (c) host launches of the same empty kernel, stream-ordered, for comparison
#include <cstdio>
#include <cuda_runtime.h>
__device__ int d_count;
__global__ void tail_chain(int left, int grid)
{
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        atomicAdd(&d_count, 1);
        if (left > 0) tail_chain<<<grid, 256, 0, cudaStreamTailLaunch>>>(left - 1, grid);
    }
}
__global__ void work(int *x) { if (threadIdx.x == 0) atomicAdd(x, 1); }
__global__ void driver(int left, int grid, int *x)
{
    if (left > 0) {
        work<<<grid, 256, 0, cudaStreamFireAndForget>>>(x);
        driver<<<1, 1, 0, cudaStreamTailLaunch>>>(left - 1, grid, x);
    }
}
__global__ void empty(int *x) { if (threadIdx.x == 0 && blockIdx.x == 0) atomicAdd(x, 1); }
int main()
{
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    int *x; cudaMalloc(&x, 4);
    for (int grid : {1, 148, 1184}) {
        const int N = 1000;
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(a);
            tail_chain<<<grid, 256>>>(N - 1, grid);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("tail chain grid=%4d: %.2f us per launch (%s)\n", grid, 1e3 * ms / N, cudaGetErrorString(cudaGetLastError()));
            cudaEventRecord(a);
            driver<<<1, 1>>>(N, grid, x);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("driver+F&F grid=%4d: %.2f us per step (%s)\n", grid, 1e3 * ms / N, cudaGetErrorString(cudaGetLastError()));
            cudaEventRecord(a);
            for (int i = 0; i < N; ++i) empty<<<grid, 256>>>(x);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("host launches grid=%4d: %.2f us per launch\n", grid, 1e3 * ms / N);
        }
    }
    int h; cudaMemcpyFromSymbol(&h, d_count, 4);
    printf("count %d\n", h);
    return 0;
}
