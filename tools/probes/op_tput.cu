// op_tput.cu -- development probe: SM-wide throughput (cycles per warp-instruction
// per SM) of the ops the irregular ranker uses, 16 warps per SM, independent chains.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
template <int OP>
__global__ void __launch_bounds__(512, 1) k(uint32_t seed, unsigned long long* cyc, uint32_t* sink) {
    __shared__ uint32_t sm[8192];
    const int lane = threadIdx.x & 31;
    uint32_t a[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) a[i] = seed * (threadIdx.x + 1) + i * 0x9E3779B9u;
    for (int i = threadIdx.x; i < 8192; i += 512) sm[i] = i * seed;
    __syncthreads();
    const long long c0 = clock64();
    constexpr int N = 256;
#pragma unroll 4
    for (int it = 0; it < N; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            if (OP == 0) a[i] = __ballot_sync(0xffffffffu, (a[i] & 1u) != 0u) ^ a[i] * 3u;
            if (OP == 1) a[i] = __popc(a[i]) + a[i] * 3u;
            if (OP == 2) a[i] = __shfl_sync(0xffffffffu, a[i], (lane + 1) & 31) + 1u;
            if (OP == 3) a[i] = sm[(threadIdx.x * 4 + (a[i] & 4) * 32 + i * 32) & 8191] + a[i];
            if (OP == 4) { sm[(threadIdx.x + i * 512 + it) & 8191] = a[i]; a[i] = a[i] * 5u + 1u; }
            if (OP == 5) a[i] = a[i] * 3u + (a[i] >> 3);
        }
    }
    __syncthreads();
    const long long c1 = clock64();
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) s ^= a[i];
    if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
    if (s == 0x1234567u) sink[0] = s + sm[lane];
}
int main() {
    unsigned long long* cyc; uint32_t* sink;
    cudaMalloc(&cyc, 148 * 8); cudaMalloc(&sink, 4);
    const char* names[] = {"VOTE(ballot)+2 alu", "POPC+2 alu", "SHFL.IDX+1 alu", "LDS+1 alu", "STS+2 alu", "3 alu (ref)"};
    auto run = [&](int op, auto kern) {
        kern<<<148, 512>>>(7u, cyc, sink);
        cudaDeviceSynchronize();
        unsigned long long h[148];
        cudaMemcpy(h, cyc, 148 * 8, cudaMemcpyDeviceToHost);
        double m = 0; for (int i = 0; i < 148; ++i) m += h[i];
        m /= 148;
        printf("%-22s %6.2f SM-cycles per warp-op (16 warps x 8 x 256 ops)\n", names[op], m / (16.0 * 8 * 256));
    };
    run(0, k<0>); run(1, k<1>); run(2, k<2>); run(3, k<3>); run(4, k<4>); run(5, k<5>);
    return 0;
}
