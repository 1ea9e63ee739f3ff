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

// The count board's reader (the fused alternative to the NCCL all-gather of
// the counts): wait until every rank's word for this call (slot 2r + tag%2,
// written by that rank's DS kernel straight into this GPU's board) carries the
// call's tag, then write all counts (d_counts, optional) and this shard's
// offset + the global total.  Acquire at system scope pairs with the writers'
// release; the two slots per rank let a rank publish call k+1 while a slower
// peer still reads call k.
__global__ void board_offsets_kernel(const uint64_t* board, uint32_t world, uint32_t rank, uint64_t tag,
                                     uint64_t* counts, uint64_t* out) {
    if (threadIdx.x != 0) return;
    unsigned long long off = 0, tot = 0;
    const uint64_t want = tag & kBoardTagMask;
    SpinGuard guard;
    for (uint32_t r = 0; r < world; ++r) {
        const uint64_t* slot = board + 2 * r + (tag & 1);
        uint64_t v;
        uint32_t ns = 32;
        while (true) {
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(slot) : "memory");
            if ((v >> kBoardCountBits) == want) break;
            guard.check("count board wait");
            __nanosleep(ns);
            ns = ns < 1024 ? 2 * ns : 1024;
        }
        const uint64_t c = v & ((1ull << kBoardCountBits) - 1);
        if (counts) counts[r] = c;
        tot += c;
        if (r < rank) off += c;
    }
    out[0] = off;
    out[1] = tot;
}

// An empty shard launches no DS kernel, so its count (0) is published here.
__global__ void publish_zero_kernel(uint64_t* const* boards, uint32_t world, uint32_t rank, uint64_t tag) {
    const uint32_t r = threadIdx.x;
    if (r < world) {
        uint64_t* slot = boards[r] + 2 * rank + (tag & 1);
        asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(slot), "l"(board_word(0, tag)) : "memory");
    }
}

// Partition's second step ("move the false elements from the
// auxiliary buffer to the tail of Array, once the true elements have been
// shifted"): dst_base[*d_offset + j] = src[j] for j < n_total - *d_offset.
// Grid-stride, one word per thread per iteration (coalesced on both sides).
__global__ void tail_copy_kernel(uint32_t* dst_base, const uint64_t* d_offset, const uint32_t* src,
                                 uint64_t n_total) {
    // Partition's second step: the falses, in order, from aux to ptr[off, n).
    // Destination-aligned 16-byte stores; the source is read as 4 coalesced
    // words per chunk (its phase relative to the destination is arbitrary).
    const uint64_t off = *d_offset;
    const uint64_t cnt = n_total - off;
    uint32_t* dst = dst_base + off;
    uint64_t head = (4u - uint32_t(reinterpret_cast<uintptr_t>(dst) >> 2)) & 3u;
    if (head > cnt) head = cnt;
    const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
    if (tid < head) dst[tid] = src[tid];
    const uint64_t nchunks = (cnt - head) >> 2;
    uint4* d4 = reinterpret_cast<uint4*>(dst + head);
    const uint32_t* s4 = src + head;
    constexpr int kU = 4;
    for (uint64_t c0 = tid; c0 < nchunks; c0 += kU * nth) {
        uint4 v[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const uint64_t c = c0 + u * nth;
            if (c < nchunks) {
                const uint32_t* q = s4 + 4 * c;
                v[u] = make_uint4(__ldg(q), __ldg(q + 1), __ldg(q + 2), __ldg(q + 3));
            }
        }
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const uint64_t c = c0 + u * nth;
            if (c < nchunks) d4[c] = v[u];
        }
    }
    const uint64_t rest = head + 4 * nchunks;
    if (tid < cnt - rest) dst[rest + tid] = src[rest + tid];
}

}  // namespace

cudaError_t launch_tail_copy(uint32_t* dst_base, const uint64_t* d_offset, const uint32_t* src,
                             const uint64_t* /*d_count_false*/, size_t n_total, cudaStream_t s) {
    count_launch();
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint64_t blocks = (n_total + 255) / 256;
    if (blocks > uint64_t(sms) * 8) blocks = uint64_t(sms) * 8;
    if (blocks == 0) blocks = 1;
    tail_copy_kernel<<<uint32_t(blocks), 256, 0, s>>>(dst_base, d_offset, src, n_total);
    return cudaGetLastError();
}

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

cudaError_t launch_board_offsets(const uint64_t* d_board, size_t world, size_t rank, uint64_t tag,
                                 uint64_t* d_counts, uint64_t* d_result, cudaStream_t s) {
    count_launch();
    board_offsets_kernel<<<1, 32, 0, s>>>(d_board, uint32_t(world), uint32_t(rank), tag, d_counts, d_result);
    return cudaGetLastError();
}

cudaError_t launch_publish_zero(uint64_t* const* d_boards, size_t world, size_t rank, uint64_t tag,
                                cudaStream_t s) {
    count_launch();
    publish_zero_kernel<<<1, uint32_t((world + 31) / 32 * 32), 0, s>>>(d_boards, uint32_t(world), uint32_t(rank), tag);
    return cudaGetLastError();
}

}  // namespace ds
