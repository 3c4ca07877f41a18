// Cluster barrier latency on B200: one cluster of C CTAs x T threads runs N
// barrier.cluster arrive.release / wait.acquire pairs (optionally with a DSMEM
// load per thread in between).  nvcc -gencode arch=compute_100a,code=sm_100a -o cluster_bar cluster_bar.cu
#include <cstdio>
#include <cuda_runtime.h>
__global__ void bar_kernel(int n, int dsm, unsigned *out)
{
    extern __shared__ unsigned sm[];
    unsigned rank, nr;
    asm("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    asm("mov.u32 %0, %%cluster_nctarank;" : "=r"(nr));
    sm[threadIdx.x] = threadIdx.x;
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    unsigned a = (unsigned)__cvta_generic_to_shared(sm + threadIdx.x), rem;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(rem) : "r"(a), "r"((rank + 1) % nr));
    unsigned acc = 0;
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) {
        if (dsm) {
            unsigned v;
            asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(rem) : "memory");
            acc += v;
        }
        asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    }
    long long t1 = clock64();
    if (threadIdx.x == 0 && rank == 0) out[0] = (unsigned)((t1 - t0) / n);
    if (acc == 12345) out[1] = acc;
}
int main()
{
    unsigned *d;
    cudaMalloc(&d, 8);
    cudaFuncSetAttribute(bar_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    for (int C : {2, 4, 8, 16})
        for (int T : {128, 512, 1024})
            for (int dsm : {0, 1}) {
                cudaLaunchConfig_t cfg = {};
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = C;
                at[0].val.clusterDim.y = 1;
                at[0].val.clusterDim.z = 1;
                cfg.gridDim = dim3(C);
                cfg.blockDim = dim3(T);
                cfg.dynamicSmemBytes = 4096;
                cfg.attrs = at;
                cfg.numAttrs = 1;
                cudaEvent_t a, b;
                cudaEventCreate(&a);
                cudaEventCreate(&b);
                cudaLaunchKernelEx(&cfg, bar_kernel, 1000, dsm, d);
                cudaEventRecord(a);
                cudaLaunchKernelEx(&cfg, bar_kernel, 10000, dsm, d);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
                float ms;
                cudaEventElapsedTime(&ms, a, b);
                unsigned h[2];
                cudaMemcpy(h, d, 8, cudaMemcpyDeviceToHost);
                printf("C=%2d T=%4d dsm=%d: %u cycles/barrier (clock64), %.3f us/barrier (events) %s\n", C, T, dsm, h[0],
                       ms * 1e3 / 10000, cudaGetErrorString(cudaGetLastError()));
            }
    return 0;
}
