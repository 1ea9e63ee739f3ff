// ds_shard.cu -- the two tiny device steps of the sharded (multi-GPU) path
// (DESIGN.md §6).  Each GPU slides its own contiguous shard with the
// single-GPU kernels; NCCL all-gathers 8-byte values between these calls.
#include "ds_device.cuh"
#include "ds_internal.h"

namespace ds {
namespace {

// Halo entry of a shard for unique across shard boundaries (R18):
// (n > 0) << 32 | ptr[n-1].  ptr[n-1] is never changed by unique.
__global__ void halo_entry_kernel(const uint32_t* ptr, uint64_t n, uint64_t* d_entry) {
    d_entry[0] = n ? ((1ull << 32) | ptr[n - 1]) : 0ull;
}

// Exclusive prefix of the all-gathered per-shard kept counts: this shard's
// global output offset and the global total.
__global__ void shard_offsets_kernel(const uint64_t* counts, uint32_t world, uint32_t rank,
                                     uint64_t* out) {
    __shared__ unsigned long long s_off, s_tot;
    if (threadIdx.x == 0) { s_off = 0; s_tot = 0; }
    __syncthreads();
    for (uint32_t r = threadIdx.x; r < world; r += blockDim.x) {
        const unsigned long long c = counts[r];
        atomicAdd(&s_tot, c);
        if (r < rank) atomicAdd(&s_off, c);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        out[0] = s_off;
        out[1] = s_tot;
    }
}

}  // namespace

cudaError_t launch_halo_entry(const uint32_t* ptr, size_t n, uint64_t* d_entry, cudaStream_t s) {
    count_launch();
    halo_entry_kernel<<<1, 1, 0, s>>>(ptr, n, d_entry);
    return cudaGetLastError();
}

cudaError_t launch_shard_offsets(const uint64_t* d_counts, size_t world, size_t rank,
                                 uint64_t* d_result, cudaStream_t s) {
    count_launch();
    shard_offsets_kernel<<<1, 128, 0, s>>>(d_counts, uint32_t(world), uint32_t(rank), d_result);
    return cudaGetLastError();
}

}  // namespace ds
