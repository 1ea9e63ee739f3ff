// launch_probe.cu -- development probe: device time of an (almost) empty
// persistent-style kernel launched right after an ordinary kernel, as a
// function of its dynamic shared memory and block size (carveout switches).
#include <cstdio>
#include <cuda_runtime.h>
__global__ void busy(float* p, size_t n) {
    for (size_t i = blockIdx.x * size_t(blockDim.x) + threadIdx.x; i < n; i += size_t(gridDim.x) * blockDim.x) p[i] = p[i] * 1.0001f + 1.f;
}
__global__ void tiny(int* out) {
    __shared__ int s0;
    if (threadIdx.x == 0) { s0 = blockIdx.x; out[blockIdx.x] = s0; }
}
int main() {
    float* p; int* o;
    const size_t n = 64 << 20;
    cudaMalloc(&p, n * 4); cudaMalloc(&o, 4096);
    cudaFuncSetAttribute(tiny, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int smems[] = {0, 16 << 10, 48 << 10, 100 << 10, 160 << 10, 198 << 10, 220 << 10};
    const int threads[] = {128, 896};
    for (int th : threads)
        for (int sm : smems) {
            float best = 1e9, sum = 0;
            for (int r = 0; r < 12; ++r) {
                busy<<<148 * 4, 256>>>(p, n);
                cudaEventRecord(a);
                tiny<<<148, th, sm>>>(o);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b);
                if (r >= 2) { best = ms < best ? ms : best; sum += ms; }
            }
            // back to back (no carveout switch in between)
            cudaEventRecord(a);
            for (int r = 0; r < 20; ++r) tiny<<<148, th, sm>>>(o);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms2; cudaEventElapsedTime(&ms2, a, b);
            printf("threads %4d smem %6d B: after busy kernel min %6.2f us mean %6.2f us | back-to-back %6.2f us/launch\n",
                   th, sm, best * 1e3, sum / 10 * 1e3, ms2 * 1e3 / 20);
        }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
