// ds_internal.h -- host-side interface between the C ABI (ds_api.cu) and the
// kernel launchers (ds_irregular.cu, ds_regular.cu, ds_shard.cu).
#pragma once

#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

namespace ds {

// Per-(device, stream) workspace: tile status words + ticket/epoch word.
struct Workspace {
    uint64_t* status = nullptr;  // [cap_tiles]
    size_t cap_tiles = 0;
    uint64_t* ctrl = nullptr;    // {epoch:32 | ticket:32}
    uint64_t launches = 0;       // launches since the status array was zeroed
};

enum class IrregOp : int { Compact = 0, Select = 1, Unique = 2 };

struct IrregArgs {
    uint32_t* ptr;
    size_t n;
    IrregOp op;
    int predicate;      // Select
    uint32_t value;     // Compact: remove value; Select: param
    const uint64_t* halo;  // Unique
    size_t halo_len;
    uint64_t* d_out_n;  // may be null
    uint32_t* out_true = nullptr;   // kept / true words (null: in place at ptr)
    uint32_t* out_false = nullptr;  // false words in input order (null: dropped)
    bool wide = false;              // 8-byte elements: n counts words (2 per element)
    uint32_t value_hi = 0;          // high word of the 8-byte value / parameter
    // Peer publication of the kept count (sharded path): the final tile also
    // writes board_word(count, tag) into slot (2*rank + tag%2) of every rank's
    // count board (peer memory over NVLink / IPC); null = none.
    uint64_t* const* pub_boards = nullptr;  // DEVICE array of `pub_world` board pointers
    uint32_t pub_world = 0, pub_rank = 0;
    uint64_t pub_tag = 0;
};

// Count-board word: {tag:28 | count:36}; a reader waits until the tag matches.
constexpr int kBoardCountBits = 36;
constexpr uint64_t kBoardTagMask = (1ull << 28) - 1;
__host__ __device__ inline uint64_t board_word(uint64_t count, uint64_t tag) {
    return ((tag & kBoardTagMask) << kBoardCountBits) | (count & ((1ull << kBoardCountBits) - 1));
}

struct RegArgs {
    uint32_t* ptr;
    uint64_t rows;
    uint64_t cols_w;      // words per row before
    uint64_t new_cols_w;  // words per row after
    uint32_t words_per_elem;
    uint32_t fill[4];
    bool pad;             // true: pad (expand, descending), false: unpad
    uint64_t src0_w = 0;       // slide: source word offset (unpad geometry with Cw == NCw)
    uint64_t out_words_w = 0;  // slide: output words (0: rows * new_cols_w)
};

// 1- and 2-byte elements whose rows are not whole words (ds_regular_bytes.cu).
struct RegBytesArgs {
    uint8_t* ptr;
    uint64_t rows;
    uint64_t cols_b;      // bytes per row before
    uint64_t new_cols_b;  // bytes per row after
    uint32_t elem_bytes;  // 1 or 2
    uint8_t fill[2];
    bool pad;
};

// Tile sizes of the kernel families (ds_tile_size).
size_t irregular_tile_words();
size_t regular_tile_words();
size_t regular_bytes_tile_bytes();

// Tiles a launch of each kernel family needs (for workspace sizing).
size_t irregular_tiles(const IrregArgs& a);
size_t regular_tiles(const RegArgs& a);

// Enqueue the kernels; return the cudaError_t of the launch.
cudaError_t launch_irregular(const IrregArgs& a, Workspace& ws, cudaStream_t s);
cudaError_t launch_regular(const RegArgs& a, Workspace& ws, cudaStream_t s);
size_t regular_bytes_tiles(const RegBytesArgs& a);
cudaError_t launch_regular_bytes(const RegBytesArgs& a, Workspace& ws, cudaStream_t s);
// Copies n words src[0, n) -> dst_base[*d_offset + j] (partition's tail move).
cudaError_t launch_tail_copy(uint32_t* dst_base, const uint64_t* d_offset, const uint32_t* src,
                             const uint64_t* d_count_false, size_t n_total, cudaStream_t s);
cudaError_t launch_halo_entry(const uint32_t* ptr, size_t n, uint64_t* d_entry, cudaStream_t s);
cudaError_t launch_shard_offsets(const uint64_t* d_counts, size_t world, size_t rank,
                                 uint64_t* d_result, cudaStream_t s);
cudaError_t launch_publish_zero(uint64_t* const* d_boards, size_t world, size_t rank, uint64_t tag,
                                cudaStream_t s);
cudaError_t launch_board_offsets(const uint64_t* d_board, size_t world, size_t rank, uint64_t tag,
                                 uint64_t* d_counts, uint64_t* d_result, cudaStream_t s);

void count_launch();
// Diagnostics buffer set by ds_debug_set_trace (null unless it covers ntiles).
uint64_t* debug_trace(size_t ntiles);

}  // namespace ds
