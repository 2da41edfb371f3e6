// Shared-memory dependent-load latency under a full grid (B200): 148 CTAs x 512 threads, one
// CTA per SM with ~200 KB of dynamic shared memory, each thread a chain of dependent LDS.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/lds lds.cu
#include <cstdio>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(512, 1) k_chain(int *out, long long *cyc, int steps, int words, int stride) {
    extern __shared__ int s[];
    for (int i = threadIdx.x; i < words; i += blockDim.x) s[i] = (int)(((long long)i * stride + 7) % words);
    __syncthreads();
    int x = (threadIdx.x * 37) % words;
    long long t0 = clock64();
    for (int k = 0; k < steps; ++k) x = s[x];
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * blockDim.x + threadIdx.x] = x;
}
__global__ void __launch_bounds__(512, 1) k_gen(int *out, long long *cyc, int steps, int words) {
    extern __shared__ int s[];
    for (int i = threadIdx.x; i < words; i += blockDim.x) s[i] = (i * 131 + 7) % words;
    __syncthreads();
    int *volatile gp = s;  // generic pointer (forces LD generic)
    int *p = gp;
    int x = (threadIdx.x * 37) % words;
    long long t0 = clock64();
    for (int k = 0; k < steps; ++k) x = p[x];
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * blockDim.x + threadIdx.x] = x;
}
int main() {
    int *out;
    long long *cyc, h[148];
    cudaMalloc(&out, 148 * 512 * 4);
    cudaMalloc(&cyc, 148 * 8);
    const int smem = 200 * 1024, words = smem / 4, steps = 1000;
    cudaFuncSetAttribute(k_chain, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(k_gen, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int stride : {1, 131, 4096}) {
        k_chain<<<148, 512, smem>>>(out, cyc, steps, words, stride);
        cudaDeviceSynchronize();
        cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
        printf("LDS chain stride %5d: %.1f cycles/load (CTA 0)\n", stride, (double)h[0] / steps);
    }
    k_gen<<<148, 512, smem>>>(out, cyc, steps, words);
    cudaDeviceSynchronize();
    cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
    printf("generic-pointer chain: %.1f cycles/load\n", (double)h[0] / steps);
    printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
}
