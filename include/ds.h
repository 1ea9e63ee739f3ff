/*
 * ds.h -- libds: in-place Data Sliding (DS) primitives on NVIDIA B200 (sm_100a).
 *
 * C ABI of the hot path.  Every call runs hand-written CUDA kernels; there is
 * no CPU fallback.  "P:NN" cites line NN of the paper text PAPER.md
 * (Gomez-Luna, Chang, Sung, Hwu, Guil, "In-Place Data Sliding Algorithms for
 * Many-Core Architectures", ICPP 2015).  Readings "Rnn" are listed in
 * DESIGN.md section 3.
 *
 * Common contract
 *  - Pointers named `ptr` are DEVICE memory on the CURRENT CUDA device
 *    (cudaMalloc'd or a torch tensor's data_ptr()), owned by the caller.
 *    libds never frees, reallocates or keeps them, and never allocates
 *    an n-sized scratch buffer (the operations are in place).
 *  - `ptr` must be 4-byte aligned; 16-byte alignment is not required.
 *  - Words are 32-bit; compact/select/unique compare bit patterns (R13),
 *    so they serve int32, uint32 and float32 arrays alike.
 *  - All argument validation happens BEFORE anything is launched: on any
 *    DS_ERROR_INVALID_VALUE / DS_ERROR_UNSUPPORTED return the buffer and
 *    the output count are untouched.  DS_ERROR_CUDA means a CUDA call
 *    failed after launch; the buffer content is then undefined (in place).
 *  - Reads: the kernels stage data with 16-byte TMA bulk copies.  A copy
 *    may start up to 12 bytes BEFORE ptr (the words before ptr in ptr's own
 *    16-byte-aligned chunk, which lie in the same allocation because device
 *    allocations start 256-byte aligned); their values are never used or
 *    written.  Nothing past the end of the caller's buffer is read: the last
 *    partial chunk of an array is loaded word by word (compact / select /
 *    unique / partition), and a pad / unpad / slide tile whose chunk would
 *    pass the end of the buffer (pad: rows*new_cols elements, unpad and
 *    slide: the sources) is gathered element by element.  Checked by
 *    compute-sanitizer memcheck with arrays that end at their allocation's
 *    end (tests/test_sanitizer_gpu.py).
 *  - Writes: only the output positions of the operation (and the fill cells
 *    of pad); never a word outside them.
 *  - Ordering between tiles (R10, "no memory fence is really
 *    required"): a tile's status word is a RELAXED store and the look-back /
 *    window polls are RELAXED loads.  The hazards are write-after-read only
 *    (no tile reads data another tile wrote; unique's boundary word is
 *    value-identical), and both sides are dependency-ordered: a tile's
 *    aggregate is computed from the words it loaded, so the status store
 *    cannot issue before those loads returned; a successor's store
 *    addresses are computed from the statuses it read, so its stores cannot
 *    issue before those loads returned.  The formal release/acquire build
 *    (libds_strict.so, -DDS_STRICT_ORDER) costs ~23 % on this hardware and is
 *    kept for testing; both builds pass the delay-injection stress at full
 *    size (tests/test_stress_gpu.py).
 *  - Kept outputs are stable.  Words in [out_n, n) (compact/select/
 *    unique) and in [rows*new_cols, rows*cols) elements (unpad) are left
 *    exactly as they were (R5).
 *  - The plain forms run on the legacy default stream and BLOCK until the
 *    result (and *out_n) is known.  The _ex forms are asynchronous and
 *    stream-ordered on `stream`; their count is written to DEVICE memory
 *    (d_out_n, may be NULL).
 *  - libds keeps, per (device, stream), a small workspace: one 64-bit
 *    status word per tile of 8192 words (one per 64-byte line, ~0.2% of
 *    the data) and one ticket/epoch word.  Calls that share a stream share it; calls on
 *    different streams may run concurrently.  ds_release_workspaces()
 *    frees it (call only when no libds kernel is in flight).  The key is
 *    the stream handle, and CUDA may hand a destroyed stream's handle to a
 *    new stream: synchronise a stream that ran libds calls before
 *    destroying it, or a new stream could share its workspace while those
 *    calls are still running.
 *  - CUDA graphs: once a stream's workspace exists (after one call on it),
 *    the _ex forms on that stream may be captured: they do not synchronise
 *    or allocate, and every launch re-arms its own ticket word (R24).  The
 *    host zeroes the status words every 2^25 launches it issues; a graph
 *    replayed more than 2^25 times should be re-captured.
 *  - Thread-safe: host state (workspaces, launch parameters) is protected
 *    by a mutex held only while a call validates and enqueues its kernels.
 *    Every blocking call reads its count through a count word of its own
 *    (taken from a per-device pool), and its read-back and stream
 *    synchronisation run without the mutex, so concurrent blocking calls
 *    never share a count and do not stall other threads' calls.
 */
#ifndef LIBDS_DS_H
#define LIBDS_DS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Same object as cudaStream_t / CUstream; NULL = legacy default stream. */
typedef struct CUstream_st* ds_stream_t;

typedef enum ds_status {
    DS_SUCCESS = 0,
    DS_ERROR_INVALID_VALUE = 1, /* NULL pointer, misaligned ptr, bad sizes  */
    DS_ERROR_UNSUPPORTED = 2,   /* valid but not implemented (ds_slide with
                                   elem_bytes 1/2, n >= 2^36 words, rows longer
                                   than 2^30 words) */
    DS_ERROR_OUT_OF_MEMORY = 3, /* workspace allocation failed              */
    DS_ERROR_CUDA = 4           /* a CUDA runtime call failed               */
} ds_status;

/* Select predicates (Fig. 11's example "element value is even",
 * P:238).  ds_select KEEPS the words for which the predicate is TRUE (R14);
 * "remove if p" is the complementary id.  `param` is a 32-bit pattern.   */
typedef enum ds_predicate {
    DS_PRED_NONZERO = 0,    /* w != 0 (bitwise)                                */
    DS_PRED_I32_GT = 1,     /* (int32)w >  (int32)param                       */
    DS_PRED_I32_NOT_GT = 2, /* !((int32)w > (int32)param)                     */
    DS_PRED_F32_GT = 3,     /* (float)w >  (float)param; NaN -> false (R16)   */
    DS_PRED_F32_NOT_GT = 4, /* !((float)w > (float)param); NaN -> true        */
    DS_PRED_I32_EVEN = 5,   /* (int32)w is even                               */
    DS_PRED_I32_ODD = 6,    /* (int32)w is odd                                */
    DS_PRED_COUNT = 7
} ds_predicate;

/* ---------------------------------------------------------------------
 * Regular DS (Algorithm 1)
 * ------------------------------------------------------------------- */

/* ds_pad -- padding matrix columns in place.
 * ptr: row-major rows x cols matrix of elem_bytes-sized elements, in a
 *      buffer the CALLER made at least rows*new_cols*elem_bytes long ("the
 *      extra memory space needs to be previously allocated adjacent to the
 *      matrix"; cannot be checked, R4).
 * After the call ptr holds rows x new_cols: row i moved forward by
 * (new_cols-cols)*i elements ("row i will be shifted by C x i") and
 * followed by new_cols-cols fill elements (zero bytes, R1/R2).
 * Requires new_cols >= cols; elem_bytes in {1, 2, 4, 8, 16}.  ptr must be
 * aligned to min(elem_bytes, 4).  1- and 2-byte elements whose rows are
 * not whole 32-bit words run on a byte-granular variant of the same kernel
 * (SURVEY 8(f)-4); rows longer than 2^30 words return DS_ERROR_UNSUPPORTED. */
ds_status ds_pad(void* ptr, size_t rows, size_t cols, size_t new_cols,
                 size_t elem_bytes);

/* ds_unpad -- "removes the extra columns": keeps the first
 * new_cols elements of every row; rows move backward.  new_cols <= cols.  */
ds_status ds_unpad(void* ptr, size_t rows, size_t cols, size_t new_cols,
                   size_t elem_bytes);

/* Asynchronous forms.  fill: HOST pointer to elem_bytes bytes copied into
 * every new cell (NULL = zero bytes).                                    */
ds_status ds_pad_ex(void* ptr, size_t rows, size_t cols, size_t new_cols,
                    size_t elem_bytes, const void* fill, ds_stream_t stream);
ds_status ds_unpad_ex(void* ptr, size_t rows, size_t cols, size_t new_cols,
                      size_t elem_bytes, ds_stream_t stream);

/* ds_slide -- the one-group regular DS: "groups of consecutive input array
 * elements are shifted by a constant amount of memory positions",
 * here a single group moved backward by `shift` elements in place:
 * elements [shift, n) of ptr move to [0, n - shift), order kept; elements
 * [n - shift, n) keep their old bytes (R5).  Same tiles, LOADED windows and
 * kernel as ds_unpad (Algorithm 1).  Requires shift <= n;
 * elem_bytes in {4, 8, 16}.  Used by the multi-GPU rebalance (DESIGN.md
 * section 5) to close a shard's gap after its head was sent to a lower
 * rank.                                                                  */
ds_status ds_slide(void* ptr, size_t n, size_t shift, size_t elem_bytes);
ds_status ds_slide_ex(void* ptr, size_t n, size_t shift, size_t elem_bytes,
                      ds_stream_t stream);

/* ---------------------------------------------------------------------
 * Irregular DS (Algorithm 2)
 * ------------------------------------------------------------------- */

/* ds_compact -- stream compaction: removes the words equal
 * (bitwise) to remove_value, keeps the others in order at ptr[0, *out_n).
 * out_n: HOST pointer, required.                                         */
ds_status ds_compact(void* ptr, size_t n, uint32_t remove_value, size_t* out_n);

/* ds_select -- select with predicate_id (ds_predicate) and
 * param = 0; keeps predicate-true words at ptr[0, *out_n).               */
ds_status ds_select(void* ptr, size_t n, int predicate_id, size_t* out_n);

/* ds_unique -- unique: word i is kept iff i == 0 or
 * w[i] != w[i-1] (bitwise, original values, R13).                 */
ds_status ds_unique(void* ptr, size_t n, size_t* out_n);

/* Asynchronous forms; d_out_n: DEVICE pointer receiving the kept count
 * (uint64), or NULL.                                                     */
ds_status ds_compact_ex(void* ptr, size_t n, uint32_t remove_value,
                        uint64_t* d_out_n, ds_stream_t stream);
ds_status ds_select_ex(void* ptr, size_t n, int predicate_id, uint32_t param,
                       uint64_t* d_out_n, ds_stream_t stream);
/* d_halo / halo_len: for a shard of a longer array (R18).  DEVICE array of
 * halo_len entries made by ds_halo_entry() for the shards BEFORE this one,
 * in order; word 0 is compared with the last word of the nearest non-empty
 * earlier shard (kept if there is none).  NULL/0 for a whole array.      */
ds_status ds_unique_ex(void* ptr, size_t n, const uint64_t* d_halo,
                       size_t halo_len, uint64_t* d_out_n, ds_stream_t stream);

/* ---------------------------------------------------------------------
 * 8-byte elements (int64 / float64; the paper evaluates pad/unpad in double,
 * P:220).  Same semantics as the 32-bit calls with n, values, counts
 * in 8-byte ELEMENTS and equality on the 64-bit pattern (R13).  ptr must be
 * 8-byte aligned.  ds_select64 takes the ds_predicate ids with the element
 * type widened: I32_* compare as int64, F32_* as double (NaN -> false for
 * GT, R16), EVEN/ODD test bit 0.  No shard halo for ds_unique64: its first
 * element is always kept.
 * ------------------------------------------------------------------- */
ds_status ds_compact64(void* ptr, size_t n, uint64_t remove_value, size_t* out_n);
ds_status ds_select64(void* ptr, size_t n, int predicate_id, size_t* out_n);
ds_status ds_unique64(void* ptr, size_t n, size_t* out_n);
ds_status ds_compact64_ex(void* ptr, size_t n, uint64_t remove_value,
                          uint64_t* d_out_n, ds_stream_t stream);
ds_status ds_select64_ex(void* ptr, size_t n, int predicate_id, uint64_t param,
                         uint64_t* d_out_n, ds_stream_t stream);
ds_status ds_unique64_ex(void* ptr, size_t n, uint64_t* d_out_n, ds_stream_t stream);

/* ---------------------------------------------------------------------
 * Partition and out-of-place variants
 * ------------------------------------------------------------------- */

/* ds_partition -- stable partition: predicate-true words first,
 * then the false words, both in input order.  As in the paper, the false
 * words go through an auxiliary buffer ("Array_false should be an
 * auxiliary buffer"): `aux` is a caller-owned DEVICE buffer of at
 * least n words, not overlapping ptr[0, n) (DS_ERROR_INVALID_VALUE
 * otherwise); libds allocates nothing n-sized.  One DS pass slides the
 * trues in place and writes the falses to aux in order, then a copy moves
 * them to the tail ptr[*out_n_true, n); aux[0, n - *out_n_true) is
 * overwritten.  out_n_true: HOST, required.                              */
ds_status ds_partition(void* ptr, size_t n, int predicate_id, void* aux, size_t* out_n_true);
/* Asynchronous form; d_out_n_true (DEVICE, required) receives the true count. */
ds_status ds_partition_ex(void* ptr, size_t n, int predicate_id, uint32_t param, void* aux,
                          uint64_t* d_out_n_true, ds_stream_t stream);

/* ds_select_copy_ex -- out-of-place select ("DS Copy_if"):
 * the predicate-true words of in[0, n) are written in order to out[0, count);
 * in is not modified.  out == in gives the in-place select; otherwise the
 * two n-word ranges must not overlap (DS_ERROR_INVALID_VALUE).           */
ds_status ds_select_copy_ex(const void* in, size_t n, int predicate_id, uint32_t param,
                            void* out, uint64_t* d_out_n, ds_stream_t stream);

/* ds_partition_copy_ex -- out-of-place stable partition: trues to
 * out_true[0, t), falses to out_false[0, n - t); in is not modified; the
 * three n-word ranges must not overlap (DS_ERROR_INVALID_VALUE).
 * d_out_n_true: DEVICE, may be NULL.                                     */
ds_status ds_partition_copy_ex(const void* in, size_t n, int predicate_id, uint32_t param,
                               void* out_true, void* out_false, uint64_t* d_out_n_true,
                               ds_stream_t stream);

/* ---------------------------------------------------------------------
 * Sharding helpers (multi-GPU).  Each GPU slides its
 * own contiguous shard; NCCL all-gathers 8-byte values between the calls.
 * ------------------------------------------------------------------- */

/* d_entry[0] = (n > 0) << 32 | ptr[n-1]  -- the shard's halo entry for
 * unique.  May be called before or after ds_unique_ex on the same shard:
 * unique never changes ptr[n-1] (it is either untouched tail or kept).   */
ds_status ds_halo_entry(const void* ptr, size_t n, uint64_t* d_entry,
                        ds_stream_t stream);

/* d_result[0] = sum(d_counts[0 .. rank)), d_result[1] = sum(d_counts[0 ..
 * world)): this shard's global output offset and the global out_n.       */
ds_status ds_shard_offsets(const uint64_t* d_counts, size_t world, size_t rank,
                           uint64_t* d_result, ds_stream_t stream);

/* Count boards: the fused alternative to the NCCL all-gather of the counts
 * (DESIGN.md section 5).  Every rank owns a board of 2*world 64-bit words in
 * its GPU's memory; every rank maps every other rank's board (CUDA IPC; peer
 * memory over NVLink between GPUs).  The DS kernel of a shard writes its kept
 * count, tagged with the call's `tag`, into slot 2*rank + tag%2 of EVERY
 * board directly from its final tile (a release store per rank, no extra
 * launch); ds_shard_offsets_board waits on the local board until every rank's
 * word carries the tag.  A rank may run at most one call ahead of another
 * (the two slots); tags must increase by one per call, starting at 1, and
 * the words hold {tag:28 | count:36}.                                      */
#define DS_IPC_HANDLE_BYTES 64
typedef struct ds_publish {
    uint64_t* const* d_boards; /* DEVICE array of `world` board pointers    */
    size_t world;
    size_t rank;
    uint64_t tag;
} ds_publish;
ds_status ds_board_alloc(size_t world, uint64_t** d_board);   /* zeroed      */
ds_status ds_board_free(uint64_t* d_board);
ds_status ds_board_ipc_handle(const uint64_t* d_board, void* handle /* DS_IPC_HANDLE_BYTES */);
ds_status ds_board_ipc_open(const void* handle, uint64_t** d_peer_board);
ds_status ds_board_ipc_close(uint64_t* d_peer_board);
/* The _ex calls plus the publication of the count (pub: HOST pointer).    */
ds_status ds_compact_pub_ex(void* ptr, size_t n, uint32_t remove_value, uint64_t* d_out_n,
                            const ds_publish* pub, ds_stream_t stream);
ds_status ds_select_pub_ex(void* ptr, size_t n, int predicate_id, uint32_t param,
                           uint64_t* d_out_n, const ds_publish* pub, ds_stream_t stream);
ds_status ds_unique_pub_ex(void* ptr, size_t n, const uint64_t* d_halo, size_t halo_len,
                           uint64_t* d_out_n, const ds_publish* pub, ds_stream_t stream);
/* d_result as ds_shard_offsets; d_counts (DEVICE, may be NULL) receives all
 * ranks' counts.                                                          */
ds_status ds_shard_offsets_board(const uint64_t* d_board, size_t world, size_t rank, uint64_t tag,
                                 uint64_t* d_counts, uint64_t* d_result, ds_stream_t stream);

/* ---------------------------------------------------------------------
 * Utilities
 * ------------------------------------------------------------------- */
const char* ds_status_string(ds_status status);
/* Message of the last failing CUDA call in this thread ("" if none).     */
const char* ds_last_error(void);
/* Frees every workspace of the calling process (all devices/streams).    */
ds_status ds_release_workspaces(void);
/* Number of kernel launches libds issued in this process (for bench.py). */
uint64_t ds_launch_count(void);
/* Diagnostics: while set, every DS kernel launch whose tile count fits
 * `capacity_tiles` records 16 uint64 per tile into the DEVICE buffer d_trace
 * (globaltimer ns: 0 drawn, 1 landed, 2 aggregate published, 3 look-back
 * start, 4 prefix published, 5 stores start, 6 stores issued; 7 SM id;
 * 8 look-back rounds, 9 polls, 10 first round read, 11 resolved, 12 the
 * bulk engine has read the stored region (irregular; region released);
 * 13 the producer starts waiting for a free input stage, 14 after the
 * ranker barrier, 15 compacted; 7 also carries bit 16 = compacted into the
 * output ring (else in place)).  When capacity_tiles also covers the grid
 * (ntiles + number of CTAs), the irregular kernels record per-CTA events in
 * the words after the tiles' (CTA b at tile index ntiles + b: 0 entry,
 * 1 set up, 2 producer done, 3/4 storer groups done, 5/6 ranker groups done,
 * 7.. resolvers done, 15 SM id; tools/trace_cta.py).
 * NULL disables.  Development aid for DESIGN.md §7, not used by the API.  */
ds_status ds_debug_set_trace(uint64_t* d_trace, size_t capacity_tiles);
/* Library version, major*10000 + minor*100 + patch.                      */
int ds_version(void);

/* Tile size of a kernel family, for tests that aim at tile edges: the
 * irregular kernel's input tile and the regular kernel's output tile in
 * 4-byte words, the byte-granular regular kernel's output tile in bytes for
 * outputs of 64 MiB or more (16384 bytes below; 0 for an unknown id).  Tiles start at the 16-byte boundary at or below
 * ptr, so tile k covers words [16B-aligned base + kT, ...).              */
typedef enum ds_kernel {
    DS_KERNEL_IRREGULAR = 0,      /* compact / select / unique / partition */
    DS_KERNEL_REGULAR = 1,        /* pad / unpad / slide, whole words      */
    DS_KERNEL_REGULAR_BYTES = 2   /* pad / unpad, 1- and 2-byte rows       */
} ds_kernel;
size_t ds_tile_size(int kernel);

#ifdef __cplusplus
}
#endif
#endif /* LIBDS_DS_H */
