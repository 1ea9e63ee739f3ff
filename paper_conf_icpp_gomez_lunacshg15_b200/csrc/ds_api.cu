// ds_api.cu -- the libds C ABI (include/ds.h): argument validation, the
// per-(device, stream) workspace cache, dispatch to the kernels, and the
// blocking wrappers.  Every validation happens before anything touches the
// device, so an error return leaves the caller's buffer untouched.
#include <cuda_runtime.h>

#include <atomic>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "ds.h"
#include "ds_device.cuh"
#include "ds_internal.h"

namespace {

constexpr uint64_t kMaxWords = (1ull << 36) - 1;     // status count field (36 bits)
constexpr uint64_t kMaxRowWords = (1ull << 30);      // 32-bit in-tile column math
constexpr uint64_t kMaxMatrixWords = (1ull << 42);   // tile ids stay 32-bit
constexpr uint64_t kResetEvery = 1ull << 25;         // zero statuses before the 26-bit epoch wraps

std::mutex g_mu;
std::map<std::pair<int, uintptr_t>, ds::Workspace> g_ws;

// Count words of the blocking forms: each call takes its own (device word,
// pinned host mirror) pair from a per-device pool, so concurrent blocking
// calls never share a count, and the read-back + stream sync run without
// the lock (other threads' asynchronous calls are not stalled by it).
struct CountSlot {
    uint64_t* d = nullptr;
    uint64_t* h = nullptr;
};
std::map<int, std::vector<CountSlot>> g_count_pool;  // free slots per device (g_mu)
std::vector<std::pair<int, CountSlot>> g_count_all;   // every slot ever made (release)
std::atomic<uint64_t> g_launches{0};
std::atomic<uint64_t*> g_trace{nullptr};
std::atomic<size_t> g_trace_cap{0};
thread_local std::string g_err;

ds_status fail(cudaError_t e, const char* what) {
    g_err = std::string(what) + ": " + cudaGetErrorString(e);
    return DS_ERROR_CUDA;
}

bool misaligned(const void* p, uintptr_t a) { return (reinterpret_cast<uintptr_t>(p) & (a - 1)) != 0; }

// Do the n-word ranges at a and b share a byte?  (n <= kMaxWords, so no overflow.)
bool overlap(const void* a, const void* b, size_t n) {
    const uintptr_t x = reinterpret_cast<uintptr_t>(a), y = reinterpret_cast<uintptr_t>(b);
    return n > 0 && x < y + 4 * n && y < x + 4 * n;
}

// Caller holds g_mu.
ds_status get_workspace(size_t tiles, cudaStream_t s, ds::Workspace** out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return fail(e, "cudaGetDevice");
    ds::Workspace& ws = g_ws[{dev, reinterpret_cast<uintptr_t>(s)}];
    if (!ws.ctrl) {
        // ctrl = {epoch 1, ticket 0}.  Nothing is kept unless every step succeeds,
        // so a failed first call leaves no half-built workspace behind.
        uint64_t* ctrl = nullptr;
        if ((e = cudaMalloc(&ctrl, sizeof(uint64_t))) != cudaSuccess)
            return e == cudaErrorMemoryAllocation ? DS_ERROR_OUT_OF_MEMORY : fail(e, "cudaMalloc");
        const uint64_t init = 1ull << 32;
        if ((e = cudaMemcpy(ctrl, &init, sizeof(init), cudaMemcpyHostToDevice)) != cudaSuccess) {
            cudaFree(ctrl);
            return fail(e, "cudaMemcpy");
        }
        ws.ctrl = ctrl;
    }
    if (ws.cap_tiles < tiles) {
        if (ws.status) {
            // The old array may still be read by queued kernels of this stream.
            if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return fail(e, "cudaStreamSynchronize");
            cudaFree(ws.status);
            ws.status = nullptr;
            ws.cap_tiles = 0;
        }
        size_t cap = tiles < 1024 ? 1024 : tiles;
        if ((e = cudaMalloc(&ws.status, cap * ds::kStatusStride * sizeof(uint64_t))) != cudaSuccess) {
            ws.status = nullptr;
            return e == cudaErrorMemoryAllocation ? DS_ERROR_OUT_OF_MEMORY : fail(e, "cudaMalloc");
        }
        ws.cap_tiles = cap;
        ws.launches = kResetEvery;  // force the zeroing below
    }
    if (ws.launches >= kResetEvery) {
        if ((e = cudaMemsetAsync(ws.status, 0, ws.cap_tiles * ds::kStatusStride * sizeof(uint64_t), s)) !=
            cudaSuccess)
            return fail(e, "cudaMemsetAsync");
        ws.launches = 0;
    }
    ws.launches++;
    *out = &ws;
    return DS_SUCCESS;
}

// Caller holds g_mu.
ds_status take_count_slot(CountSlot* out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return fail(e, "cudaGetDevice");
    std::vector<CountSlot>& pool = g_count_pool[dev];
    if (!pool.empty()) {
        *out = pool.back();
        pool.pop_back();
        return DS_SUCCESS;
    }
    CountSlot c;
    if ((e = cudaMalloc(&c.d, sizeof(uint64_t))) != cudaSuccess)
        return e == cudaErrorMemoryAllocation ? DS_ERROR_OUT_OF_MEMORY : fail(e, "cudaMalloc");
    if ((e = cudaMallocHost(&c.h, sizeof(uint64_t))) != cudaSuccess) {
        cudaFree(c.d);
        return e == cudaErrorMemoryAllocation ? DS_ERROR_OUT_OF_MEMORY : fail(e, "cudaMallocHost");
    }
    g_count_all.push_back({dev, c});
    *out = c;
    return DS_SUCCESS;
}

void give_count_slot(const CountSlot& c) {
    std::lock_guard<std::mutex> lock(g_mu);
    for (const auto& kv : g_count_all)
        if (kv.second.d == c.d) {
            g_count_pool[kv.first].push_back(c);
            return;
        }
}

// Reads a blocking call's count back (legacy default stream) without the lock.
ds_status read_count(const CountSlot& c, size_t* out_n) {
    cudaError_t e = cudaMemcpyAsync(c.h, c.d, sizeof(uint64_t), cudaMemcpyDeviceToHost, nullptr);
    if (e == cudaSuccess) e = cudaStreamSynchronize(nullptr);
    ds_status st = e == cudaSuccess ? DS_SUCCESS : fail(e, "count read-back");
    if (st == DS_SUCCESS) *out_n = size_t(*c.h);
    give_count_slot(c);
    return st;
}

ds_status run_irregular(const ds::IrregArgs& a, cudaStream_t s) {
    std::lock_guard<std::mutex> lock(g_mu);
    ds::Workspace* ws = nullptr;
    ds_status st = get_workspace(ds::irregular_tiles(a), s, &ws);
    if (st != DS_SUCCESS) return st;
    cudaError_t e = ds::launch_irregular(a, *ws, s);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "irregular kernel launch");
}

ds_status check_irregular(const void* ptr, size_t n, const uint64_t* d_out_n) {
    if (n > 0 && ptr == nullptr) return DS_ERROR_INVALID_VALUE;
    if (misaligned(ptr, 4) || misaligned(d_out_n, 8)) return DS_ERROR_INVALID_VALUE;
    if (n > kMaxWords) return DS_ERROR_UNSUPPORTED;
    return DS_SUCCESS;
}

ds_status irregular_ex(ds::IrregArgs a, cudaStream_t s) {
    if (a.n == 0) {
        if (a.d_out_n) {
            cudaError_t e = cudaMemsetAsync(a.d_out_n, 0, sizeof(uint64_t), s);
            if (e != cudaSuccess) return fail(e, "cudaMemsetAsync");
        }
        if (a.pub_boards) {  // an empty shard still publishes its count
            cudaError_t e = ds::launch_publish_zero(a.pub_boards, a.pub_world, a.pub_rank, a.pub_tag, s);
            if (e != cudaSuccess) return fail(e, "publish launch");
        }
        return DS_SUCCESS;
    }
    return run_irregular(a, s);
}

// Peer publication of a shard's count (count boards).
ds_status apply_publish(const ds_publish* pub, ds::IrregArgs* a) {
    if (!pub) return DS_ERROR_INVALID_VALUE;
    if (!pub->d_boards || pub->world == 0 || pub->world > 1024 || pub->rank >= pub->world)
        return DS_ERROR_INVALID_VALUE;
    if (misaligned(pub->d_boards, 8)) return DS_ERROR_INVALID_VALUE;
    a->pub_boards = pub->d_boards;
    a->pub_world = uint32_t(pub->world);
    a->pub_rank = uint32_t(pub->rank);
    a->pub_tag = pub->tag;
    return DS_SUCCESS;
}

// Blocking form: legacy default stream, count read back through the
// workspace's pinned mirror.
ds_status irregular_blocking(ds::IrregArgs a, size_t* out_n) {
    if (a.n == 0) {
        *out_n = 0;
        return DS_SUCCESS;
    }
    CountSlot slot;
    ds_status st;
    {
        std::lock_guard<std::mutex> lock(g_mu);
        st = take_count_slot(&slot);
        if (st != DS_SUCCESS) return st;
        ds::Workspace* ws = nullptr;
        st = get_workspace(ds::irregular_tiles(a), nullptr, &ws);
        if (st == DS_SUCCESS) {
            a.d_out_n = slot.d;
            cudaError_t e = ds::launch_irregular(a, *ws, nullptr);
            if (e != cudaSuccess) st = fail(e, "irregular kernel launch");
        }
    }
    if (st != DS_SUCCESS) {
        give_count_slot(slot);
        return st;
    }
    return read_count(slot, out_n);
}

ds_status run_regular(const ds::RegArgs& a, cudaStream_t s);

// Sub-word elements (eb 1, 2): rows of whole words run on the word kernel
// (the fill replicated into a word); anything else on the byte kernel.
ds_status run_sub_word(void* ptr, size_t rows, size_t cols, size_t new_cols, size_t eb, bool pad,
                       const void* fill, cudaStream_t s) {
    if (pad ? new_cols < cols : new_cols > cols) return DS_ERROR_INVALID_VALUE;
    size_t big = pad ? new_cols : cols, tmp = 0;
    if (__builtin_mul_overflow(rows, big, &tmp) || __builtin_mul_overflow(tmp, eb, &tmp))
        return DS_ERROR_INVALID_VALUE;
    if (tmp > 0 && ptr == nullptr) return DS_ERROR_INVALID_VALUE;
    if (misaligned(ptr, eb)) return DS_ERROR_INVALID_VALUE;
    if (uint64_t(big) * eb >= kMaxRowWords) return DS_ERROR_UNSUPPORTED;
    if (tmp / 4 > kMaxMatrixWords) return DS_ERROR_UNSUPPORTED;
    uint8_t f[2] = {0, 0};
    if (fill) std::memcpy(f, fill, eb);
    if (eb == 1) f[1] = f[0];
    const uint64_t cb = uint64_t(cols) * eb, ncb = uint64_t(new_cols) * eb;
    if (rows == 0 || cb == ncb || ncb == 0) return DS_SUCCESS;  // nothing moves
    if (cb % 4 == 0 && ncb % 4 == 0 && !misaligned(ptr, 4)) {
        ds::RegArgs a{};
        a.ptr = static_cast<uint32_t*>(ptr);
        a.rows = rows;
        a.cols_w = cb / 4;
        a.new_cols_w = ncb / 4;
        a.words_per_elem = 1;
        a.pad = pad;
        const uint32_t w = uint32_t(f[0]) | uint32_t(f[1]) << 8;
        a.fill[0] = a.fill[1] = a.fill[2] = a.fill[3] = w | w << 16;
        return run_regular(a, s);
    }
    ds::RegBytesArgs b{};
    b.ptr = static_cast<uint8_t*>(ptr);
    b.rows = rows;
    b.cols_b = cb;
    b.new_cols_b = ncb;
    b.elem_bytes = uint32_t(eb);
    b.fill[0] = f[0];
    b.fill[1] = f[1];
    b.pad = pad;
    std::lock_guard<std::mutex> lock(g_mu);
    ds::Workspace* ws = nullptr;
    ds_status st = get_workspace(ds::regular_bytes_tiles(b), s, &ws);
    if (st != DS_SUCCESS) return st;
    cudaError_t e = ds::launch_regular_bytes(b, *ws, s);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "regular bytes kernel launch");
}

ds_status check_regular(const void* ptr, size_t rows, size_t cols, size_t new_cols, size_t eb,
                        bool pad, ds::RegArgs* a) {
    if (eb != 4 && eb != 8 && eb != 16) return DS_ERROR_INVALID_VALUE;
    if (pad ? new_cols < cols : new_cols > cols) return DS_ERROR_INVALID_VALUE;
    size_t big = pad ? new_cols : cols, tmp = 0;
    if (__builtin_mul_overflow(rows, big, &tmp) || __builtin_mul_overflow(tmp, eb, &tmp))
        return DS_ERROR_INVALID_VALUE;
    if (tmp > 0 && ptr == nullptr) return DS_ERROR_INVALID_VALUE;
    if (misaligned(ptr, 4)) return DS_ERROR_INVALID_VALUE;
    const uint64_t w = eb / 4;
    if (uint64_t(big) * w >= kMaxRowWords) return DS_ERROR_UNSUPPORTED;
    if (tmp / 4 > kMaxMatrixWords) return DS_ERROR_UNSUPPORTED;
    a->ptr = static_cast<uint32_t*>(const_cast<void*>(ptr));
    a->rows = rows;
    a->cols_w = uint64_t(cols) * w;
    a->new_cols_w = uint64_t(new_cols) * w;
    a->words_per_elem = uint32_t(w);
    a->pad = pad;
    std::memset(a->fill, 0, sizeof(a->fill));
    return DS_SUCCESS;
}

ds_status run_regular(const ds::RegArgs& a, cudaStream_t s) {
    // No-ops: nothing moves and no fill cell exists / nothing is kept.
    if (a.rows == 0 || a.cols_w == a.new_cols_w || a.new_cols_w == 0) return DS_SUCCESS;
    std::lock_guard<std::mutex> lock(g_mu);
    ds::Workspace* ws = nullptr;
    ds_status st = get_workspace(ds::regular_tiles(a), s, &ws);
    if (st != DS_SUCCESS) return st;
    cudaError_t e = ds::launch_regular(a, *ws, s);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "regular kernel launch");
}

// ---- 8-byte elements (n counts elements; the kernels see 2n words) ----
ds_status check_wide(const void* ptr, size_t n, const uint64_t* d_out_n) {
    if (n > 0 && ptr == nullptr) return DS_ERROR_INVALID_VALUE;
    if (misaligned(ptr, 8) || misaligned(d_out_n, 8)) return DS_ERROR_INVALID_VALUE;
    if (n > kMaxWords / 2) return DS_ERROR_UNSUPPORTED;
    return DS_SUCCESS;
}

ds::IrregArgs wide_args(void* ptr, size_t n, ds::IrregOp op, int pred, uint64_t value, uint64_t* d_out_n) {
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), 2 * n, op, pred, uint32_t(value), nullptr, 0, d_out_n};
    a.wide = true;
    a.value_hi = uint32_t(value >> 32);
    return a;
}

ds_status wide_blocking(ds::IrregArgs a, size_t* out_n) {
    size_t words = 0;
    ds_status st = irregular_blocking(a, &words);  // the kernel reports elements already
    if (st == DS_SUCCESS) *out_n = words;
    return st;
}

ds_status sync_default() {
    cudaError_t e = cudaStreamSynchronize(nullptr);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "cudaStreamSynchronize");
}

}  // namespace

namespace ds {
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
uint64_t* debug_trace(size_t ntiles) { return ntiles <= g_trace_cap.load() ? g_trace.load() : nullptr; }
}  // namespace ds

extern "C" {

ds_status ds_pad_ex(void* ptr, size_t rows, size_t cols, size_t new_cols, size_t elem_bytes,
                    const void* fill, ds_stream_t stream) {
    if (elem_bytes == 1 || elem_bytes == 2)
        return run_sub_word(ptr, rows, cols, new_cols, elem_bytes, true, fill,
                            reinterpret_cast<cudaStream_t>(stream));
    ds::RegArgs a{};
    ds_status st = check_regular(ptr, rows, cols, new_cols, elem_bytes, true, &a);
    if (st != DS_SUCCESS) return st;
    if (fill) std::memcpy(a.fill, fill, elem_bytes);
    return run_regular(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_unpad_ex(void* ptr, size_t rows, size_t cols, size_t new_cols, size_t elem_bytes,
                      ds_stream_t stream) {
    if (elem_bytes == 1 || elem_bytes == 2)
        return run_sub_word(ptr, rows, cols, new_cols, elem_bytes, false, nullptr,
                            reinterpret_cast<cudaStream_t>(stream));
    ds::RegArgs a{};
    ds_status st = check_regular(ptr, rows, cols, new_cols, elem_bytes, false, &a);
    if (st != DS_SUCCESS) return st;
    return run_regular(a, reinterpret_cast<cudaStream_t>(stream));
}

// The blocking forms synchronise only when a kernel was enqueued (a no-op
// call needs no device).
ds_status ds_pad(void* ptr, size_t rows, size_t cols, size_t new_cols, size_t elem_bytes) {
    ds_status st = ds_pad_ex(ptr, rows, cols, new_cols, elem_bytes, nullptr, nullptr);
    if (st != DS_SUCCESS || rows == 0 || cols == new_cols) return st;
    return sync_default();
}

ds_status ds_unpad(void* ptr, size_t rows, size_t cols, size_t new_cols, size_t elem_bytes) {
    ds_status st = ds_unpad_ex(ptr, rows, cols, new_cols, elem_bytes, nullptr);
    if (st != DS_SUCCESS || rows == 0 || cols == new_cols || new_cols == 0) return st;
    return sync_default();
}

ds_status ds_slide_ex(void* ptr, size_t n, size_t shift, size_t elem_bytes, ds_stream_t stream) {
    if (elem_bytes == 1 || elem_bytes == 2) return DS_ERROR_UNSUPPORTED;
    if (elem_bytes != 4 && elem_bytes != 8 && elem_bytes != 16) return DS_ERROR_INVALID_VALUE;
    if (shift > n) return DS_ERROR_INVALID_VALUE;
    size_t bytes = 0;
    if (__builtin_mul_overflow(n, elem_bytes, &bytes)) return DS_ERROR_INVALID_VALUE;
    if (n > 0 && ptr == nullptr) return DS_ERROR_INVALID_VALUE;
    if (misaligned(ptr, 4)) return DS_ERROR_INVALID_VALUE;
    if (bytes / 4 > kMaxMatrixWords) return DS_ERROR_UNSUPPORTED;
    if (shift == 0 || shift == n) return DS_SUCCESS;  // nothing moves
    // A regular DS with one group: unpad geometry with equal row lengths and
    // a source offset (rows of kSlideRow words; any length works).
    constexpr uint64_t kSlideRow = 1ull << 20;
    const uint64_t w = elem_bytes / 4;
    ds::RegArgs a{};
    a.ptr = static_cast<uint32_t*>(ptr);
    a.out_words_w = uint64_t(n - shift) * w;
    a.src0_w = uint64_t(shift) * w;
    a.cols_w = a.new_cols_w = kSlideRow;
    a.rows = (a.out_words_w + kSlideRow - 1) / kSlideRow;
    a.words_per_elem = uint32_t(w);
    a.pad = false;
    std::lock_guard<std::mutex> lock(g_mu);
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    ds::Workspace* ws = nullptr;
    ds_status st = get_workspace(ds::regular_tiles(a), s, &ws);
    if (st != DS_SUCCESS) return st;
    cudaError_t e = ds::launch_regular(a, *ws, s);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "regular kernel launch");
}

ds_status ds_slide(void* ptr, size_t n, size_t shift, size_t elem_bytes) {
    ds_status st = ds_slide_ex(ptr, n, shift, elem_bytes, nullptr);
    if (st != DS_SUCCESS || shift == 0 || shift == n) return st;
    return sync_default();
}

ds_status ds_compact_ex(void* ptr, size_t n, uint32_t remove_value, uint64_t* d_out_n,
                        ds_stream_t stream) {
    ds_status st = check_irregular(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Compact, 0, remove_value,
                    nullptr, 0, d_out_n};
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_select_ex(void* ptr, size_t n, int predicate_id, uint32_t param, uint64_t* d_out_n,
                       ds_stream_t stream) {
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Select, predicate_id, param,
                    nullptr, 0, d_out_n};
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_unique_ex(void* ptr, size_t n, const uint64_t* d_halo, size_t halo_len,
                       uint64_t* d_out_n, ds_stream_t stream) {
    if (halo_len > 0 && d_halo == nullptr) return DS_ERROR_INVALID_VALUE;
    if (misaligned(d_halo, 8)) return DS_ERROR_INVALID_VALUE;
    if (halo_len > 0xFFFFFFFFull) return DS_ERROR_UNSUPPORTED;
    ds_status st = check_irregular(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Unique, 0, 0u,
                    d_halo, halo_len, d_out_n};
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_compact(void* ptr, size_t n, uint32_t remove_value, size_t* out_n) {
    if (!out_n) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(ptr, n, nullptr);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Compact, 0, remove_value,
                    nullptr, 0, nullptr};
    return irregular_blocking(a, out_n);
}

ds_status ds_select(void* ptr, size_t n, int predicate_id, size_t* out_n) {
    if (!out_n) return DS_ERROR_INVALID_VALUE;
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(ptr, n, nullptr);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Select, predicate_id, 0u,
                    nullptr, 0, nullptr};
    return irregular_blocking(a, out_n);
}

ds_status ds_unique(void* ptr, size_t n, size_t* out_n) {
    if (!out_n) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(ptr, n, nullptr);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Unique, 0, 0u, nullptr, 0, nullptr};
    return irregular_blocking(a, out_n);
}

ds_status ds_select_copy_ex(const void* in, size_t n, int predicate_id, uint32_t param, void* out,
                            uint64_t* d_out_n, ds_stream_t stream) {
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(in, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    if (n > 0 && (!out || misaligned(out, 4))) return DS_ERROR_INVALID_VALUE;
    if (out != in && overlap(in, out, n)) return DS_ERROR_INVALID_VALUE;  // in place only at out == in
    ds::IrregArgs a{const_cast<uint32_t*>(static_cast<const uint32_t*>(in)), n, ds::IrregOp::Select,
                    predicate_id, param, nullptr, 0, d_out_n};
    a.out_true = static_cast<uint32_t*>(out);
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_partition_copy_ex(const void* in, size_t n, int predicate_id, uint32_t param,
                               void* out_true, void* out_false, uint64_t* d_out_n_true,
                               ds_stream_t stream) {
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(in, n, d_out_n_true);
    if (st != DS_SUCCESS) return st;
    if (n > 0 && (!out_true || !out_false || misaligned(out_true, 4) || misaligned(out_false, 4)))
        return DS_ERROR_INVALID_VALUE;
    if (overlap(in, out_true, n) || overlap(in, out_false, n) || overlap(out_true, out_false, n))
        return DS_ERROR_INVALID_VALUE;
    ds::IrregArgs a{const_cast<uint32_t*>(static_cast<const uint32_t*>(in)), n, ds::IrregOp::Select,
                    predicate_id, param, nullptr, 0, d_out_n_true};
    a.out_true = static_cast<uint32_t*>(out_true);
    a.out_false = static_cast<uint32_t*>(out_false);
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_partition_ex(void* ptr, size_t n, int predicate_id, uint32_t param, void* aux,
                          uint64_t* d_out_n_true, ds_stream_t stream) {
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    if (!d_out_n_true) return DS_ERROR_INVALID_VALUE;  // the tail copy needs the true count
    ds_status st = check_irregular(ptr, n, d_out_n_true);
    if (st != DS_SUCCESS) return st;
    if (n > 0 && (!aux || misaligned(aux, 4))) return DS_ERROR_INVALID_VALUE;
    if (overlap(ptr, aux, n)) return DS_ERROR_INVALID_VALUE;
    if (n == 0) return irregular_ex(ds::IrregArgs{static_cast<uint32_t*>(ptr), 0, ds::IrregOp::Select,
                                                  predicate_id, param, nullptr, 0, d_out_n_true},
                                    reinterpret_cast<cudaStream_t>(stream));
    // Step 1 (one DS pass): trues slide in place, falses go to aux in order.
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Select, predicate_id, param,
                    nullptr, 0, d_out_n_true};
    a.out_false = static_cast<uint32_t*>(aux);
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    st = run_irregular(a, s);
    if (st != DS_SUCCESS) return st;
    // Step 2: aux[0, n - n_true) -> ptr[n_true, n).
    cudaError_t e = ds::launch_tail_copy(static_cast<uint32_t*>(ptr), d_out_n_true,
                                         static_cast<const uint32_t*>(aux), nullptr, n, s);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "tail copy launch");
}

ds_status ds_partition(void* ptr, size_t n, int predicate_id, void* aux, size_t* out_n_true) {
    if (!out_n_true) return DS_ERROR_INVALID_VALUE;
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(ptr, n, nullptr);
    if (st != DS_SUCCESS) return st;
    if (n > 0 && (!aux || misaligned(aux, 4))) return DS_ERROR_INVALID_VALUE;
    if (overlap(ptr, aux, n)) return DS_ERROR_INVALID_VALUE;
    if (n == 0) {
        *out_n_true = 0;
        return DS_SUCCESS;
    }
    // The true count goes to this call's own count word: the DS pass writes it
    // and the tail copy reads it, so no other call may share it.
    CountSlot slot;
    {
        std::lock_guard<std::mutex> lock(g_mu);
        st = take_count_slot(&slot);
        if (st != DS_SUCCESS) return st;
    }
    st = ds_partition_ex(ptr, n, predicate_id, 0u, aux, slot.d, nullptr);
    if (st != DS_SUCCESS) {
        give_count_slot(slot);
        return st;
    }
    return read_count(slot, out_n_true);
}

ds_status ds_compact_pub_ex(void* ptr, size_t n, uint32_t remove_value, uint64_t* d_out_n,
                            const ds_publish* pub, ds_stream_t stream) {
    ds_status st = check_irregular(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Compact, 0, remove_value, nullptr, 0, d_out_n};
    if ((st = apply_publish(pub, &a)) != DS_SUCCESS) return st;
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_select_pub_ex(void* ptr, size_t n, int predicate_id, uint32_t param, uint64_t* d_out_n,
                           const ds_publish* pub, ds_stream_t stream) {
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_irregular(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Select, predicate_id, param, nullptr, 0, d_out_n};
    if ((st = apply_publish(pub, &a)) != DS_SUCCESS) return st;
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_unique_pub_ex(void* ptr, size_t n, const uint64_t* d_halo, size_t halo_len, uint64_t* d_out_n,
                           const ds_publish* pub, ds_stream_t stream) {
    if (halo_len > 0 && d_halo == nullptr) return DS_ERROR_INVALID_VALUE;
    if (misaligned(d_halo, 8)) return DS_ERROR_INVALID_VALUE;
    if (halo_len > 0xFFFFFFFFull) return DS_ERROR_UNSUPPORTED;
    ds_status st = check_irregular(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    ds::IrregArgs a{static_cast<uint32_t*>(ptr), n, ds::IrregOp::Unique, 0, 0u, d_halo, halo_len, d_out_n};
    if ((st = apply_publish(pub, &a)) != DS_SUCCESS) return st;
    return irregular_ex(a, reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_board_alloc(size_t world, uint64_t** d_board) {
    if (!d_board || world == 0 || world > 1024) return DS_ERROR_INVALID_VALUE;
    uint64_t* b = nullptr;
    cudaError_t e = cudaMalloc(&b, 2 * world * sizeof(uint64_t));
    if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? DS_ERROR_OUT_OF_MEMORY : fail(e, "cudaMalloc");
    if ((e = cudaMemset(b, 0, 2 * world * sizeof(uint64_t))) != cudaSuccess) {
        cudaFree(b);
        return fail(e, "cudaMemset");
    }
    *d_board = b;
    return DS_SUCCESS;
}

ds_status ds_board_free(uint64_t* d_board) {
    if (!d_board) return DS_SUCCESS;
    cudaError_t e = cudaFree(d_board);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "cudaFree");
}

ds_status ds_board_ipc_handle(const uint64_t* d_board, void* handle) {
    if (!d_board || !handle) return DS_ERROR_INVALID_VALUE;
    cudaIpcMemHandle_t h;
    cudaError_t e = cudaIpcGetMemHandle(&h, const_cast<uint64_t*>(d_board));
    if (e != cudaSuccess) return fail(e, "cudaIpcGetMemHandle");
    static_assert(sizeof(h) == DS_IPC_HANDLE_BYTES, "IPC handle size");
    std::memcpy(handle, &h, sizeof(h));
    return DS_SUCCESS;
}

ds_status ds_board_ipc_open(const void* handle, uint64_t** d_peer_board) {
    if (!handle || !d_peer_board) return DS_ERROR_INVALID_VALUE;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, sizeof(h));
    void* ptr = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return fail(e, "cudaIpcOpenMemHandle");
    *d_peer_board = static_cast<uint64_t*>(ptr);
    return DS_SUCCESS;
}

ds_status ds_board_ipc_close(uint64_t* d_peer_board) {
    if (!d_peer_board) return DS_ERROR_INVALID_VALUE;
    cudaError_t e = cudaIpcCloseMemHandle(d_peer_board);
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "cudaIpcCloseMemHandle");
}

ds_status ds_shard_offsets_board(const uint64_t* d_board, size_t world, size_t rank, uint64_t tag,
                                 uint64_t* d_counts, uint64_t* d_result, ds_stream_t stream) {
    if (!d_board || !d_result || world == 0 || world > 1024 || rank >= world) return DS_ERROR_INVALID_VALUE;
    if (misaligned(d_board, 8) || misaligned(d_result, 8) || misaligned(d_counts, 8)) return DS_ERROR_INVALID_VALUE;
    cudaError_t e = ds::launch_board_offsets(d_board, world, rank, tag, d_counts, d_result,
                                             reinterpret_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "board offsets launch");
}

ds_status ds_halo_entry(const void* ptr, size_t n, uint64_t* d_entry, ds_stream_t stream) {
    if (!d_entry || misaligned(d_entry, 8)) return DS_ERROR_INVALID_VALUE;
    if (n > 0 && (ptr == nullptr || misaligned(ptr, 4))) return DS_ERROR_INVALID_VALUE;
    cudaError_t e = ds::launch_halo_entry(static_cast<const uint32_t*>(ptr), n, d_entry,
                                          reinterpret_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "halo entry launch");
}

ds_status ds_shard_offsets(const uint64_t* d_counts, size_t world, size_t rank, uint64_t* d_result,
                           ds_stream_t stream) {
    if (!d_counts || !d_result || world == 0 || rank >= world) return DS_ERROR_INVALID_VALUE;
    if (misaligned(d_counts, 8) || misaligned(d_result, 8)) return DS_ERROR_INVALID_VALUE;
    if (world > 0xFFFFFFFFull) return DS_ERROR_UNSUPPORTED;
    cudaError_t e = ds::launch_shard_offsets(d_counts, world, rank, d_result,
                                             reinterpret_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? DS_SUCCESS : fail(e, "shard offsets launch");
}

ds_status ds_compact64_ex(void* ptr, size_t n, uint64_t remove_value, uint64_t* d_out_n, ds_stream_t stream) {
    ds_status st = check_wide(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    return irregular_ex(wide_args(ptr, n, ds::IrregOp::Compact, 0, remove_value, d_out_n),
                        reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_select64_ex(void* ptr, size_t n, int predicate_id, uint64_t param, uint64_t* d_out_n,
                         ds_stream_t stream) {
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_wide(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    return irregular_ex(wide_args(ptr, n, ds::IrregOp::Select, predicate_id, param, d_out_n),
                        reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_unique64_ex(void* ptr, size_t n, uint64_t* d_out_n, ds_stream_t stream) {
    ds_status st = check_wide(ptr, n, d_out_n);
    if (st != DS_SUCCESS) return st;
    return irregular_ex(wide_args(ptr, n, ds::IrregOp::Unique, 0, 0, d_out_n),
                        reinterpret_cast<cudaStream_t>(stream));
}

ds_status ds_compact64(void* ptr, size_t n, uint64_t remove_value, size_t* out_n) {
    if (!out_n) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_wide(ptr, n, nullptr);
    if (st != DS_SUCCESS) return st;
    return wide_blocking(wide_args(ptr, n, ds::IrregOp::Compact, 0, remove_value, nullptr), out_n);
}

ds_status ds_select64(void* ptr, size_t n, int predicate_id, size_t* out_n) {
    if (!out_n) return DS_ERROR_INVALID_VALUE;
    if (predicate_id < 0 || predicate_id >= DS_PRED_COUNT) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_wide(ptr, n, nullptr);
    if (st != DS_SUCCESS) return st;
    return wide_blocking(wide_args(ptr, n, ds::IrregOp::Select, predicate_id, 0, nullptr), out_n);
}

ds_status ds_unique64(void* ptr, size_t n, size_t* out_n) {
    if (!out_n) return DS_ERROR_INVALID_VALUE;
    ds_status st = check_wide(ptr, n, nullptr);
    if (st != DS_SUCCESS) return st;
    return wide_blocking(wide_args(ptr, n, ds::IrregOp::Unique, 0, 0, nullptr), out_n);
}

const char* ds_status_string(ds_status s) {
    switch (s) {
    case DS_SUCCESS: return "DS_SUCCESS";
    case DS_ERROR_INVALID_VALUE: return "DS_ERROR_INVALID_VALUE";
    case DS_ERROR_UNSUPPORTED: return "DS_ERROR_UNSUPPORTED";
    case DS_ERROR_OUT_OF_MEMORY: return "DS_ERROR_OUT_OF_MEMORY";
    case DS_ERROR_CUDA: return "DS_ERROR_CUDA";
    }
    return "DS_ERROR_UNKNOWN";
}

const char* ds_last_error(void) { return g_err.c_str(); }

ds_status ds_release_workspaces(void) {
    std::lock_guard<std::mutex> lock(g_mu);
    int cur = 0;
    cudaGetDevice(&cur);
    ds_status st = DS_SUCCESS;
    for (auto& kv : g_ws) {
        ds::Workspace& ws = kv.second;
        if (cudaSetDevice(kv.first.first) != cudaSuccess) continue;
        cudaDeviceSynchronize();
        if (ws.status) cudaFree(ws.status);
        if (ws.ctrl) cudaFree(ws.ctrl);
    }
    g_ws.clear();
    for (auto& kv : g_count_all) {
        if (cudaSetDevice(kv.first) != cudaSuccess) continue;
        cudaDeviceSynchronize();
        cudaFree(kv.second.d);
        cudaFreeHost(kv.second.h);
    }
    g_count_all.clear();
    g_count_pool.clear();
    cudaSetDevice(cur);
    return st;
}

uint64_t ds_launch_count(void) { return g_launches.load(); }

ds_status ds_debug_set_trace(uint64_t* d_trace, size_t capacity_tiles) {
    if (d_trace && misaligned(d_trace, 8)) return DS_ERROR_INVALID_VALUE;
    g_trace.store(d_trace);
    g_trace_cap.store(d_trace ? capacity_tiles : 0);
    return DS_SUCCESS;
}

int ds_version(void) { return 200; }

size_t ds_tile_size(int kernel) {
    switch (kernel) {
    case DS_KERNEL_IRREGULAR: return ds::irregular_tile_words();
    case DS_KERNEL_REGULAR: return ds::regular_tile_words();
    case DS_KERNEL_REGULAR_BYTES: return ds::regular_bytes_tile_bytes();
    }
    return 0;
}

}  // extern "C"
