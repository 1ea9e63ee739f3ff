// ds_device.cuh -- device building blocks shared by the DS kernels (sm_100a).
//
//  * Dynamic tile ID allocation (the paper's Fig. 4) fused with a
//    per-launch epoch: one 64-bit word {epoch:32 | ticket:32}.  The CTA that
//    draws the LAST ticket of a launch re-arms the word for the next launch
//    (epoch+1, ticket 0) -- every ticket of this launch has been drawn by
//    then, so no memset launch is needed between calls.
//  * Tile status words (the paper's per-WG flags, Fig. 3 P:92-103 / Fig. 7
//    P:143-156) as 64-bit {state:2 | epoch:26 | count:36}.  A status whose
//    epoch differs from the launch's is "not yet published" (R8: a zero
//    count is never confused with "not ready").
//  * Release/acquire at GPU scope (R10): publish with st.release.gpu after
//    the tile's loads; poll with ld.relaxed.gpu (no L1 invalidation per
//    poll) and execute ONE fence.acq_rel.gpu once every awaited status is
//    seen.
//  * 128-bit streaming loads/stores that do not allocate in L1.
#pragma once

#include <cstdint>
#include <cstdio>

namespace ds {

constexpr uint64_t kStateShift = 62;
constexpr uint64_t kEpochShift = 36;
constexpr uint64_t kEpochMask = (1ull << 26) - 1;
constexpr uint64_t kCountMask = (1ull << 36) - 1;
constexpr uint64_t kStateAgg = 1;     // irregular: tile aggregate only
constexpr uint64_t kStateLoaded = 1;  // regular: tile's sources are loaded
constexpr uint64_t kStateIncl = 2;    // irregular: inclusive prefix known

// Status words are spread kStatusStride uint64 apart: tiles
// finishing at the same time sit on different L2 lines.
#ifndef DS_STATUS_STRIDE
#define DS_STATUS_STRIDE 8
#endif
constexpr uint64_t kStatusStride = DS_STATUS_STRIDE;
__host__ __device__ __forceinline__ uint64_t* status_ptr(uint64_t* base, int64_t tile) {
    return base + tile * int64_t(kStatusStride);
}
__host__ __device__ __forceinline__ const uint64_t* status_ptr(const uint64_t* base, int64_t tile) {
    return base + tile * int64_t(kStatusStride);
}

__host__ __device__ __forceinline__ uint64_t make_status(uint64_t state, uint64_t epoch,
                                                         uint64_t count) {
    return (state << kStateShift) | ((epoch & kEpochMask) << kEpochShift) | (count & kCountMask);
}
__device__ __forceinline__ uint32_t status_state(uint64_t s) { return uint32_t(s >> kStateShift); }
__device__ __forceinline__ uint64_t status_count(uint64_t s) { return s & kCountMask; }
__device__ __forceinline__ bool status_current(uint64_t s, uint64_t epoch) {
    return status_state(s) != 0 && ((s >> kEpochShift) & kEpochMask) == (epoch & kEpochMask);
}

__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_gpu(uint64_t* p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_gpu(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void fence_acq_rel_gpu() {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

// Status publication and the look-back's closing fence.
// The DS hazards are write-after-read only: a tile never reads data that a
// lower tile wrote (unique's boundary word is value-identical), so what must
// hold is "every read of tile j completes before any tile > j overwrites
// it".  A tile's reads have completed (the TMA transaction count reached
// zero, or the values were consumed) before its status store is even
// issued, and a successor's stores are issued only after it has read that
// status, so relaxed status words suffice physically; GPU-scope release /
// acquire fences cost ~1-2 us each here (MEMBAR.GPU drains the SM's whole
// store stream).  -DDS_STRICT_ORDER restores release stores and the acquire
// fence of the formal PTX-model argument; the test suite runs both builds.
__device__ __forceinline__ void publish_status(uint64_t* p, uint64_t v) {
#ifdef DS_STRICT_ORDER
    st_release_gpu(p, v);
#else
    st_relaxed_gpu(p, v);
#endif
}
__device__ __forceinline__ void lookback_acquire() {
#ifdef DS_STRICT_ORDER
    fence_acq_rel_gpu();
#endif
}

struct alignas(16) u32x4 {
    uint32_t x, y, z, w;
};

__device__ __forceinline__ u32x4 ldg_stream_v4(const uint32_t* p) {
    u32x4 r;
    asm volatile("ld.global.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}
__device__ __forceinline__ uint32_t ldg_stream(const uint32_t* p) {
    uint32_t r;
    asm volatile("ld.global.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
    return r;
}
__device__ __forceinline__ void stg_stream_v4(uint32_t* p, uint32_t a, uint32_t b, uint32_t c,
                                              uint32_t d) {
    asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(a),
                 "r"(b), "r"(c), "r"(d)
                 : "memory");
}
__device__ __forceinline__ void stg_stream(uint32_t* p, uint32_t a) {
    asm volatile("st.global.L1::no_allocate.u32 [%0], %1;" ::"l"(p), "r"(a) : "memory");
}

// Fig. 4: thread 0 draws the next dynamic tile id.  Returns
// {ticket, epoch}.  A launch makes exactly `draws` draws in total (the
// persistent kernels: ntiles + gridDim.x, every CTA's last draw fails); the
// CTA that makes the final draw re-arms the word for the next launch.
// Split form: issue_ticket() sends the atomic (the caller can overlap its
// round trip with other work, e.g. the barrier set-up at kernel entry);
// take_ticket() decodes it and re-arms the word after the launch's last draw.
__device__ __forceinline__ unsigned long long issue_ticket(uint64_t* ctrl) {
    return atomicAdd(reinterpret_cast<unsigned long long*>(ctrl), 1ull);
}
__device__ __forceinline__ void take_ticket(uint64_t* ctrl, uint32_t draws, unsigned long long old,
                                            uint32_t& ticket, uint32_t& epoch) {
    ticket = uint32_t(old);
    epoch = uint32_t(old >> 32);
    if (ticket == draws - 1) {
        uint32_t ne = epoch + 1;
        if ((ne & kEpochMask) == 0) ne++;  // epoch 0 is never valid (zeroed status)
        atomicExch(reinterpret_cast<unsigned long long*>(ctrl), (unsigned long long)ne << 32);
    }
}
__device__ __forceinline__ void draw_ticket(uint64_t* ctrl, uint32_t draws, uint32_t& ticket,
                                            uint32_t& epoch) {
    take_ticket(ctrl, draws, issue_ticket(ctrl), ticket, epoch);
}

// ---- shared-memory mbarrier + 1-D TMA bulk copy (cp.async.bulk) --------
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count)
                 : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
// Failure detection: with -DDS_SPIN_CAP_NS=t every wait loop of
// the kernels gives up after t ns of waiting and traps (printing where), so a
// lost publication (a bug, or DS_DEBUG_DROP_TILE) ends the launch with a CUDA
// error that the API reports as DS_ERROR_CUDA instead of hanging the process.
// Compiled out of the release library.
struct SpinGuard {
#ifdef DS_SPIN_CAP_NS
    uint64_t t0 = 0;
    __device__ __forceinline__ void check(const char* where) {
        uint64_t now;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
        if (t0 == 0) t0 = now;
        else if (now - t0 > uint64_t(DS_SPIN_CAP_NS)) {
            printf("libds: wait in %s exceeded DS_SPIN_CAP_NS (block %d thread %d)\n", where, blockIdx.x,
                   threadIdx.x);
            __trap();
        }
    }
#else
    __device__ __forceinline__ void check(const char*) {}
#endif
};

// Blocking wait for the phase with the given parity.  The suspend-time hint
// lets the hardware park the warp until the phase completes instead of
// re-issuing try_wait in a tight loop.
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity, uint32_t hint_ns);
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
#ifdef DS_SPIN_CAP_NS
    SpinGuard g;
    while (!mbar_try_wait(bar, parity, 100000u)) g.check("mbarrier wait");
    return;
#endif
#ifdef DS_MBAR_SPIN
    asm volatile(
        "{\n"
        ".reg .pred P;\n"
        "DS_WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n"
        "@!P bra DS_WAIT_%=;\n"
        "}\n" ::"r"(smem_addr(bar)),
        "r"(parity)
        : "memory");
    return;
#endif
#ifdef DS_MBAR_BACKOFF
    // Polls with a growing sleep in between (no suspend hint): fewer mbarrier
    // unit operations per wait while the TMA completes transactions on it.
    for (uint32_t ns = 32;; ns = ns < DS_MBAR_BACKOFF ? 2 * ns : ns) {
        uint32_t done;
        asm volatile(
            "{\n.reg .pred P;\n"
            "mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n"
            "selp.u32 %0, 1, 0, P;\n}\n"
            : "=r"(done)
            : "r"(smem_addr(bar)), "r"(parity)
            : "memory");
        if (done) return;
        __nanosleep(ns);
    }
#endif
    asm volatile(
        "{\n"
        ".reg .pred P;\n"
        "DS_WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1, %2;\n"
        "@!P bra DS_WAIT_%=;\n"
        "}\n" ::"r"(smem_addr(bar)),
        "r"(parity), "r"(1000000u)
        : "memory");
}
// Non-blocking probe of the phase with the given parity.
__device__ __forceinline__ bool mbar_test_wait(uint64_t* bar, uint32_t parity) {
    uint32_t done;
    asm volatile(
        "{\n.reg .pred P;\n"
        "mbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n"
        "selp.u32 %0, 1, 0, P;\n}\n"
        : "=r"(done)
        : "r"(smem_addr(bar)), "r"(parity)
        : "memory");
    return done != 0;
}
// One bounded wait (up to ~hint_ns); returns whether the phase completed.
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity, uint32_t hint_ns) {
    uint32_t done;
    asm volatile(
        "{\n.reg .pred P;\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2, %3;\n"
        "selp.u32 %0, 1, 0, P;\n}\n"
        : "=r"(done)
        : "r"(smem_addr(bar)), "r"(parity), "r"(hint_ns)
        : "memory");
    return done != 0;
}

// Named barrier among `count` threads (a subset of the CTA, whole warps).
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
// Arrive on a named barrier without waiting (producer side of a bar.arrive /
// bar.sync pair: the arriving thread's prior writes are ordered before the
// waiters' later accesses).
__device__ __forceinline__ void named_bar_arrive(uint32_t id, uint32_t count) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(count) : "memory");
}

// Global -> shared bulk copy of `bytes` (multiple of 16, both addresses
// 16-byte aligned), completing on `bar`.  Streams through L2 (evict-first).
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "{\n"
        ".reg .b64 pol;\n"
        "createpolicy.fractional.L2::evict_first.b64 pol, 1.0;\n"
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1], %2, [%3], pol;\n"
        "}\n" ::"r"(smem_addr(dst)),
        "l"(src), "r"(bytes), "r"(smem_addr(bar))
        : "memory");
}

// L2 prefetch of `bytes` (multiple of 16, 16-byte aligned) global bytes: the
// bulk engine reads them into L2 without a destination or completion.
__device__ __forceinline__ void bulk_prefetch_l2(const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}

// Shared -> global bulk copy (TMA store) of `bytes` (multiple of 16, both
// addresses 16-byte aligned), tracked by the issuing thread's bulk async-group.
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
    asm volatile(
        "{\n"
        ".reg .b64 pol;\n"
        "createpolicy.fractional.L2::evict_first.b64 pol, 1.0;\n"
        "cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, pol;\n"
        "}\n" ::"l"(dst),
        "r"(smem_addr(src)), "r"(bytes)
        : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// Wait until at most N of this thread's bulk groups still READ shared memory.
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
// Wait until every bulk group of this thread has completed (writes visible).
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ uint32_t smid() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return r;
}
// Diagnostics (ds_debug_set_trace): per-tile events, 16 words per tile.
constexpr int kTraceWords = 16;
__device__ __forceinline__ void trace_event(uint64_t* trace, uint64_t tile, int ev, uint64_t v) {
    if (trace) trace[tile * kTraceWords + ev] = v;
}

// Scheduling-stress hook (tests T3): with -DDS_DEBUG_DELAY the calling
// thread sleeps a pseudo-random 0..4 us depending on (tile, site), which
// reorders ticket -> load -> publish -> store across CTAs.  Compiled out of
// the release library.
__device__ __forceinline__ void debug_delay(uint64_t tile, uint32_t site) {
#ifdef DS_DEBUG_DELAY
    uint64_t z = tile * 0x9E3779B97F4A7C15ull + site * 0xBF58476D1CE4E5B9ull;
    z ^= z >> 31;
    z *= 0x94D049BB133111EBull;
    z ^= z >> 29;
    if ((z & 3) == 0) __nanosleep(uint32_t(z >> 40) % 4000u);
#else
    (void)tile;
    (void)site;
#endif
}

// Granlund-Montgomery round-up division by a runtime constant d (1 <= d <
// 2^31), exact for every 32-bit numerator.
struct FastDiv {
    uint32_t d, mul, shift;
};
__host__ inline FastDiv make_fastdiv(uint32_t d) {
    FastDiv f{d, 0, 0};
    uint32_t l = 0;
    while ((1ull << l) < d) ++l;
    f.shift = l;
    f.mul = uint32_t(((1ull << 32) * ((1ull << l) - d)) / d + 1);
    return f;
}
__device__ __forceinline__ uint32_t fastdiv(uint32_t n, const FastDiv& f) {
    uint64_t t = __umulhi(n, f.mul);
    return uint32_t((t + n) >> f.shift);
}

// Same for 64-bit numerators (d < 2^32): q = (t + ((n - t) >> 1)) >> (l-1),
// t = mulhi64(n, m), m = floor(2^64 (2^l - d) / d) + 1.  Exact for all n.
struct FastDiv64 {
    uint64_t d, mul;
    uint32_t shift;
};
__host__ inline FastDiv64 make_fastdiv64(uint64_t d) {
    FastDiv64 f{d, 0, 0};
    uint32_t l = 0;
    while ((1ull << l) < d) ++l;
    f.shift = l;
    if (l > 0) {
        unsigned __int128 num = (unsigned __int128)((1ull << l) - d) << 64;
        f.mul = uint64_t(num / d) + 1;
    }
    return f;
}
__device__ __forceinline__ uint64_t fastdiv64(uint64_t n, const FastDiv64& f) {
    if (f.shift == 0) return n;  // d == 1
    const uint64_t t = __umul64hi(n, f.mul);
    return (t + ((n - t) >> 1)) >> (f.shift - 1);
}

}  // namespace ds
