// bw_probe.cu -- development probe (not part of libds): HBM read / copy
// throughput of the load paths the DS kernels can use on sm_100a.
//   tma_read<S, CH>: persistent CTAs, one producer lane keeps S bulk copies of
//                    CH bytes in flight (cp.async.bulk -> smem ring), consumer
//                    warps touch one word and release the stage.
//   ldg_read:        grid-stride 128-bit loads, U independent loads per thread.
//   tma_copy<S,CH>:  bulk load + bulk store of the same chunk (read+write).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o bw_probe tools/bw_probe.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); exit(1); } } while (0)

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(c) : "memory"); }
__device__ __forceinline__ void mbar_expect(uint64_t* b, uint32_t bytes) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes) : "memory"); }
__device__ __forceinline__ void mbar_arrive(uint64_t* b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(b)) : "memory"); }
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
    asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1, %2;\n@!P bra W_%=;\n}\n" ::"r"(sa(b)), "r"(par), "r"(1000000u) : "memory");
}
__device__ __forceinline__ void g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(sa(dst)), "l"(src), "r"(bytes), "r"(sa(bar)) : "memory");
}
__device__ __forceinline__ void s2g(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(sa(src)), "r"(bytes) : "memory");
}

// S stages of CH bytes; W consumer warps.  COPY: bulk-store each chunk to dst.
template <int COPY>
__global__ void __launch_bounds__(256) tma_kernel(const char* src, char* dst, size_t nchunks, int S, int CH,
                                                 unsigned long long* sink) {
    extern __shared__ __align__(128) char sm[];
    __shared__ __align__(8) uint64_t full[32], empty[32];
    const int tid = threadIdx.x, warp = tid >> 5;
    if (tid == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (warp == 0) {
        if (tid != 0) return;
        uint32_t k = 0;
        for (size_t c = blockIdx.x; c < nchunks; c += gridDim.x, ++k) {
            const int s = k % S;
            mbar_wait(&empty[s], ((k / S) & 1) ^ 1);
            mbar_expect(&full[s], CH);
            g2s(sm + size_t(s) * CH, src + c * CH, CH, &full[s]);
        }
    } else if (warp == 1) {
        if (tid != 32) return;
        uint32_t k = 0;
        unsigned long long acc = 0;
        for (size_t c = blockIdx.x; c < nchunks; c += gridDim.x, ++k) {
            const int s = k % S;
            mbar_wait(&full[s], (k / S) & 1);
            acc += *(volatile uint32_t*)(sm + size_t(s) * CH);
            if (COPY) {
                s2g(dst + c * CH, sm + size_t(s) * CH, CH);
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            }
            mbar_arrive(&empty[s]);
        }
        if (COPY) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
        if (acc == 0x1234567) atomicAdd(sink, acc);
    }
}


// Closer to the DS irregular kernel: optional L2 evict_first policy on the
// loads (POL), dynamic chunk ids from a global atomic ticket (TICKET), and 16
// "ranker" warps that each read a 512-word segment of the stage from shared
// memory and meet at a named barrier before the stage is released (RANK).
template <int POL, int TICKET, int RANK>
__global__ void __launch_bounds__(1024) tma2_kernel(const char* src, size_t nchunks, int S, int CH,
                                                   unsigned long long* ctr, unsigned long long* sink) {
    extern __shared__ __align__(128) char sm[];
    __shared__ __align__(8) uint64_t full[32], empty[32];
    __shared__ uint32_t chunk_of[32];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (tid == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int nr = RANK ? 16 : 1;
    if (warp == 0) {
        if (tid != 0) return;
        size_t c = blockIdx.x;
        for (uint32_t k = 0;; ++k) {
            const int s = k % S;
            mbar_wait(&empty[s], ((k / S) & 1) ^ 1);
            if (TICKET) c = atomicAdd(ctr, 1ull);
            chunk_of[s] = c < nchunks ? uint32_t(c) : 0xffffffffu;
            if (c >= nchunks) { mbar_arrive(&full[s]); return; }
            mbar_expect(&full[s], CH);
            if (POL) {
                asm volatile("{\n.reg .b64 pol;\ncreatepolicy.fractional.L2::evict_first.b64 pol, 1.0;\n"
                             "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], pol;\n}\n"
                             ::"r"(sa(sm + size_t(s) * CH)), "l"(src + c * CH), "r"(CH), "r"(sa(&full[s])) : "memory");
            } else {
                g2s(sm + size_t(s) * CH, src + c * CH, CH, &full[s]);
            }
            if (!TICKET) c += gridDim.x;
        }
    } else if (warp <= nr) {
        const int rw = warp - 1;
        unsigned long long acc = 0;
        for (uint32_t k = 0;; ++k) {
            const int s = k % S;
            mbar_wait(&full[s], (k / S) & 1);
            if (chunk_of[s] == 0xffffffffu) break;
            const uint32_t* st = reinterpret_cast<const uint32_t*>(sm + size_t(s) * CH);
            if (RANK) {
                const int words = CH / 4 / 16;
                uint32_t cnt = 0;
                for (int i = lane; i < words; i += 32) cnt += __popc(__ballot_sync(0xffffffffu, st[rw * words + i] != 0));
                acc += cnt;
                asm volatile("bar.sync 1, %0;" ::"r"(16 * 32) : "memory");
                if (tid == 32) mbar_arrive(&empty[s]);
            } else {
                if (lane == 0) { acc += st[0]; mbar_arrive(&empty[s]); }
            }
        }
        if (acc == 0x1234567) atomicAdd(sink, acc);
    }
}

template <int U>
__global__ void ldg_kernel(const uint4* __restrict__ src, size_t n16, unsigned long long* sink) {
    uint32_t acc = 0;
    const size_t stride = size_t(gridDim.x) * blockDim.x;
    for (size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n16; i += stride * U) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const size_t j = i + u * stride;
            if (j < n16) asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w) : "l"(src + j));
            else v[u] = make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].w;
    }
    if (acc == 0x1234567) atomicAdd(sink, acc);
}

__global__ void gtimer_kernel(unsigned long long* out) {
    long long c0 = clock64();
    unsigned long long g = 0, acc = 0;
    for (int i = 0; i < 100; ++i) {
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g));
        acc += g;
    }
    long long c1 = clock64();
    unsigned long long g0, g1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g0));
    long long c2 = clock64();
    while (clock64() - c2 < 100000) {}
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g1));
    out[0] = (c1 - c0) / 100;
    out[1] = g1 - g0;
    out[2] = acc;
}

__global__ void flush_kernel(uint4* p, size_t n16) {
    for (size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n16; i += size_t(gridDim.x) * blockDim.x)
        p[i] = make_uint4(i, 0, 0, 0);
}

int main() {
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    const size_t bytes = size_t(4) << 30;
    char *a, *b, *fl;
    unsigned long long* sink;
    CK(cudaMalloc(&a, bytes));
    CK(cudaMalloc(&b, bytes));
    CK(cudaMalloc(&fl, size_t(512) << 20));
    CK(cudaMalloc(&sink, 8));
    CK(cudaMemset(a, 1, bytes));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto timeit = [&](const char* name, double traffic, auto launch) {
        float best = 1e30f;
        for (int r = 0; r < 5; ++r) {
            flush_kernel<<<sms * 4, 256>>>((uint4*)fl, (size_t(512) << 20) / 16);
            cudaEventRecord(e0);
            launch();
            cudaEventRecord(e1);
            CK(cudaEventSynchronize(e1));
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 1 && ms < best) best = ms;
        }
        CK(cudaGetLastError());
        printf("%-44s %8.1f us  %7.1f GB/s\n", name, best * 1e3, traffic / (best * 1e-3) / 1e9);
    };
    {
        unsigned long long h[3];
        unsigned long long* d3;
        CK(cudaMalloc(&d3, 24));
        gtimer_kernel<<<1, 1>>>(d3);
        CK(cudaMemcpy(h, d3, 24, cudaMemcpyDeviceToHost));
        printf("globaltimer read: %llu cycles each; 100000 cycles = %llu ns of globaltimer\n", h[0], h[1]);
        if (getenv("GT_ONLY")) return 0;
    }

    if (getenv("DS_LIKE")) {
        unsigned long long* ctr;
        CK(cudaMalloc(&ctr, 8));
        const int S = 6, CH = 32768;
        const size_t smem = size_t(S) * CH, nch = bytes / CH;
#define RUN2(P, T, R)                                                                                       \
        {                                                                                                  \
            CK(cudaFuncSetAttribute(tma2_kernel<P, T, R>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem))); \
            char name[96];                                                                                 \
            snprintf(name, sizeof name, "tma2 pol=%d ticket=%d rank=%d S=6 CH=32K", P, T, R);              \
            timeit(name, double(bytes), [&] {                                                              \
                cudaMemsetAsync(ctr, 0, 8);                                                                \
                tma2_kernel<P, T, R><<<sms, R ? 32 * 17 : 64, smem>>>(a, nch, S, CH, ctr, sink);           \
            });                                                                                            \
        }
        RUN2(0, 0, 0) RUN2(1, 0, 0) RUN2(0, 1, 0) RUN2(0, 0, 1) RUN2(1, 1, 1) RUN2(0, 1, 1)
        return 0;
    }
    struct Cfg { int S, CH, ctas; };
    const Cfg cfgs[] = {{6, 32768, 1}, {3, 65536, 1}, {12, 16384, 1}, {24, 8192, 1}, {6, 16384, 2}, {3, 32768, 2},
                        {12, 8192, 2}, {4, 16384, 3}, {6, 8192, 4}, {13, 16384, 1}};
    for (const Cfg& c : cfgs) {
        const size_t smem = size_t(c.S) * c.CH;
        CK(cudaFuncSetAttribute(tma_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
        CK(cudaFuncSetAttribute(tma_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
        char name[96];
        snprintf(name, sizeof name, "tma_read  S=%2d CH=%5d ctas/SM=%d", c.S, c.CH, c.ctas);
        const size_t nch = bytes / c.CH;
        timeit(name, double(bytes), [&] { tma_kernel<0><<<sms * c.ctas, 64, smem>>>(a, b, nch, c.S, c.CH, sink); });
        snprintf(name, sizeof name, "tma_copy  S=%2d CH=%5d ctas/SM=%d", c.S, c.CH, c.ctas);
        timeit(name, 2.0 * double(bytes), [&] { tma_kernel<1><<<sms * c.ctas, 64, smem>>>(a, b, nch, c.S, c.CH, sink); });
    }
    timeit("ldg_read U=4 (8 CTAs x 256 / SM)", double(bytes), [&] { ldg_kernel<4><<<sms * 8, 256>>>((const uint4*)a, bytes / 16, sink); });
    timeit("ldg_read U=8 (8 CTAs x 256 / SM)", double(bytes), [&] { ldg_kernel<8><<<sms * 8, 256>>>((const uint4*)a, bytes / 16, sink); });
    timeit("ldg_read U=8 (4 CTAs x 256 / SM)", double(bytes), [&] { ldg_kernel<8><<<sms * 4, 256>>>((const uint4*)a, bytes / 16, sink); });
    timeit("cudaMemcpy D2D", 2.0 * double(bytes), [&] { cudaMemcpyAsync(b, a, bytes, cudaMemcpyDeviceToDevice); });
    return 0;
}
