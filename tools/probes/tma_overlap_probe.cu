// Probe: does cuTensorMapEncodeTiled accept a 2-D map whose rows overlap
// (row stride 1 KB < row length 2 KB), and does a TMA store of a {256, R} box
// at an arbitrary inner coordinate write R*256 contiguous words?
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cstdio>
#include <cstdint>
#include <vector>
__global__ void k(const __grid_constant__ CUtensorMap m, int x, int y, int words) {
    extern __shared__ __align__(128) uint32_t sm[];
    for (int i = threadIdx.x; i < words; i += blockDim.x) sm[i] = 1000000 + i;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(reinterpret_cast<uint64_t>(&m)), "r"(x), "r"(y), "r"(static_cast<uint32_t>(__cvta_generic_to_shared(sm))) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
}
int main() {
    void* f = nullptr; cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
    auto enc = (PFN_cuTensorMapEncodeTiled_v12000)f;
    const size_t N = 1 << 20;
    uint32_t* d; cudaMalloc(&d, N * 4); cudaMemset(d, 0, N * 4);
    for (int R : {1, 8, 32}) {
        CUtensorMap m;
        cuuint64_t dims[2] = {512, N / 256 - 1};
        cuuint64_t strides[1] = {1024};
        cuuint32_t box[2] = {256, (cuuint32_t)R}, es[2] = {1, 1};
        CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, d, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        printf("R=%d encode -> %d\n", R, (int)r);
        if (r != CUDA_SUCCESS) continue;
        cudaMemset(d, 0, N * 4);
        int x = 37, y = 100, words = 256 * R;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, words * 4);
        k<<<1, 256, words * 4>>>(m, x, y, words);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<uint32_t> h(N);
        cudaMemcpy(h.data(), d, N * 4, cudaMemcpyDeviceToHost);
        size_t g0 = 256 * y + x; int bad = 0; size_t nz = 0;
        for (size_t i = 0; i < N; ++i) {
            uint32_t want = (i >= g0 && i < g0 + words) ? 1000000 + (i - g0) : 0;
            if (h[i] != want) ++bad;
            if (h[i]) ++nz;
        }
        printf("R=%d kernel %s, nonzero %zu (want %d), mismatches %d\n", R, cudaGetErrorString(e), nz, words, bad);
    }
    return 0;
}
