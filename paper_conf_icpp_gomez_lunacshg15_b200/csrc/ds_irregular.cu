// ds_irregular.cu -- irregular Data Sliding on sm_100a: in-place, stable
// stream compaction, select and unique (Algorithm 2, P:168-190;
// §III-B; primitives §IV-B/C P:230-282).
//
// Persistent, warp-specialised CTAs (two per SM) walk input tiles of
// T = 8192 words in dynamic-ticket order (Fig. 4) through a 3-stage
// shared-memory ring:
//
//   producer warp   a1 draw the next ticket when a stage is free
//                   a2 one TMA bulk copy of the tile (plus, for unique, the
//                      16 bytes before it) into the stage (Alg. 2 lines 1-11;
//                      P:84 "on-chip memory")
//                   a3+a4 the tile aggregate: keep flags and one warp
//                      reduction ("Reduction", done before the sync
//                      as P:158 recommends)
//                   a5a publish AGG (release) the moment the tile has landed
//   resolver warp   a5b decoupled look-back over 128 predecessors per round
//                      trip, publish INCL; the last tile writes out_n (a8).
//                      This replaces the serial flag chain of Fig. 7, which
//                      is latency-bound on B200
//   8 consumer      a6 rank of every kept word in input order ("binary
//   warps              prefix sum"): ballot/popc within each
//                      warp-vector + a scan of the 64 warp-vector counts
//                   a7 scatter kept words in the stage at their final 16-byte
//                      phase, then 128-bit stores of [excl, excl+A) (scalar
//                      head/tail), then release the stage
//
// A drawn tile's AGG depends only on its own bulk copy, never on this CTA's
// progress through earlier tiles (DESIGN.md §5 explains why that matters).
// In-place safety: AGG/INCL are published only after the
// tile's copy completed; a tile stores only after the look-back saw AGG/INCL
// of every lower tile; outputs of tile t lie in [0, (t+1)T), so no lower tile
// writes into a higher tile's input.  Deadlock freedom: look-backs wait only
// for lower (already drawn) tiles, whose AGG is published without waiting.
#include "ds_device.cuh"
#include "ds_internal.h"

namespace ds {
namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr uint32_t kNoTile = 0xffffffffu;

struct IrregParams {
    uint32_t* abase;  // 16-byte-aligned base (ptr - lo)
    uint64_t lo, hi;  // valid virtual word range [lo, hi)
    uint64_t* status;
    uint64_t* ctrl;
    uint64_t* d_out_n;
    const uint64_t* halo;
    uint32_t halo_len;
    uint32_t ntiles;
    uint32_t draws;   // ntiles + gridDim.x
    uint32_t value;   // compact: remove value; select: predicate parameter
};

// ---- predicates (a3) ----------------------------------------------------
struct OpCompact {  // remove words equal to a value
    static constexpr bool kUnique = false;
    __device__ static bool keep(uint32_t w, uint32_t v) { return w != v; }
};
template <int P>
struct OpSelect {  // keep predicate-true words (R14); ids = ds_predicate
    static constexpr bool kUnique = false;
    __device__ static bool keep(uint32_t w, uint32_t param) {
        if constexpr (P == 0) return w != 0u;
        else if constexpr (P == 1) return int32_t(w) > int32_t(param);
        else if constexpr (P == 2) return !(int32_t(w) > int32_t(param));
        else if constexpr (P == 3) return __uint_as_float(w) > __uint_as_float(param);
        else if constexpr (P == 4) return !(__uint_as_float(w) > __uint_as_float(param));
        else if constexpr (P == 5) return (w & 1u) == 0u;
        else return (w & 1u) != 0u;
    }
};
struct OpUnique {  // keep w[i] iff it differs from w[i-1]
    static constexpr bool kUnique = true;
    __device__ static bool keep(uint32_t, uint32_t) { return true; }
};

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// ---- tile geometry ------------------------------------------------------
constexpr int kConsumerWarps = 8;
constexpr int kCT = 32 * kConsumerWarps;  // consumer threads
constexpr int kItems = 32;                // words per consumer thread
constexpr int kVec = kItems / 4;
constexpr int kT = kCT * kItems;          // 8192 words = 32 KB per tile
constexpr int kSlots = kVec * kConsumerWarps;  // warp-vectors per tile (64)
constexpr int kPre = 4;                   // words before the tile (unique's boundary word)
constexpr int kStageWords = kT + kPre + 4;  // + 4: store-phase realignment slack
constexpr int kStages = 3;
constexpr int kThreads = 32 * (2 + kConsumerWarps);
constexpr size_t kSmem = size_t(kStages) * kStageWords * 4;
static_assert(kSlots == 64, "producer scan assumes two slots per lane");

// Keep mask of the 4 words of warp-vector slot x (tile word index) from the
// staged tile.  Identical in producer and consumers.
template <class Op>
__device__ __forceinline__ uint32_t keep_mask(const IrregParams& p, const uint32_t* stage,
                                              uint64_t tb, bool full, int x, const u32x4& q,
                                              bool has_hprev, uint32_t hprev) {
    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
    uint32_t m = 0;
    if constexpr (Op::kUnique) {
        uint32_t prev = stage[kPre + x - 1];  // x == 0: the word before the tile
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const uint64_t e = tb + x + k;
            bool kp = w[k] != prev;
            if (e == p.lo) kp = !has_hprev || w[k] != hprev;  // array's first word (R18)
            prev = w[k];
            if ((full || (e >= p.lo && e < p.hi)) && kp) m |= 1u << k;
        }
    } else {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const uint64_t e = tb + x + k;
            if ((full || (e >= p.lo && e < p.hi)) && Op::keep(w[k], p.value)) m |= 1u << k;
        }
    }
    return m;
}

// Shard halo (R18): last word of the nearest non-empty earlier shard.
__device__ __forceinline__ bool halo_prev(const IrregParams& p, uint32_t& prev) {
    for (uint32_t h = p.halo_len; h-- > 0;) {
        const uint64_t ent = p.halo[h];
        if (ent >> 32) {
            prev = uint32_t(ent);
            return true;
        }
    }
    return false;
}

// a5b: decoupled look-back by one warp, 4 predecessors per lane (128 per
// round trip).  Lane l, slot m examines tile base - (4l + m).  Waits only
// for the tiles up to the nearest INCL predecessor.  Ends with one acquire
// fence per lane and a __syncwarp so lane 0's later release is cumulative
// over everything the warp observed.
constexpr int kLB = 4;

__device__ __forceinline__ uint64_t lookback(const uint64_t* __restrict__ status, uint32_t tile,
                                             uint32_t epoch, int lane) {
    uint64_t excl = 0;
    int64_t base = int64_t(tile) - 1;
    while (true) {
        uint64_t s[kLB];
        uint32_t okm = 0;  // bit m: slot m has a current status
#pragma unroll
        for (int m = 0; m < kLB; ++m) {
            const int64_t idx = base - (kLB * lane + m);
            if (idx >= 0) {
                s[m] = ld_relaxed_gpu(status + idx);
                if (status_current(s[m], epoch)) okm |= 1u << m;
            } else {
                s[m] = make_status(kStateIncl, epoch, 0);  // virtual INCL(0) before tile 0
                okm |= 1u << m;
            }
        }
        uint32_t ns = 16;
        int L, M;  // nearest INCL: lane L, slot M (L == 32: none in this round)
        while (true) {
            uint32_t inclm = 0;
#pragma unroll
            for (int m = 0; m < kLB; ++m)
                if ((okm >> m & 1u) && status_state(s[m]) == kStateIncl) inclm |= 1u << m;
            const uint32_t lanes_incl = __ballot_sync(kFull, inclm != 0);
            L = lanes_incl ? __ffs(lanes_incl) - 1 : 32;
            M = __shfl_sync(kFull, inclm ? __ffs(inclm) - 1 : kLB, L & 31);
            // every slot strictly before (L, M) and (L, M) itself must be current
            const uint32_t need = lane < L ? ((1u << kLB) - 1) : (lane == L ? ((2u << M) - 1) : 0u);
            const bool bad = (okm & need) != need;
            if (!__any_sync(kFull, bad)) break;
            __nanosleep(ns);
            ns = ns < 256 ? ns * 2 : 256;
#pragma unroll
            for (int m = 0; m < kLB; ++m) {
                if (!(okm >> m & 1u) && (need >> m & 1u)) {
                    const int64_t idx = base - (kLB * lane + m);
                    s[m] = ld_relaxed_gpu(status + idx);
                    if (status_current(s[m], epoch)) okm |= 1u << m;
                }
            }
        }
        uint32_t agg = 0;
        uint64_t inc = 0;
#pragma unroll
        for (int m = 0; m < kLB; ++m) {
            if (lane < L || (lane == L && m < M)) agg += uint32_t(status_count(s[m]));
            if (lane == L && m == M) inc = status_count(s[m]);
        }
        excl += uint64_t(__reduce_add_sync(kFull, agg));
        if (L < 32) {
            excl += __shfl_sync(kFull, inc, L);
            break;
        }
        base -= 32 * kLB;
    }
    fence_acq_rel_gpu();
    __syncwarp();
    return excl;
}

struct StageMeta {
    uint32_t tile;           // kNoTile: end of this CTA's work
    uint32_t total;          // kept words in the tile
    unsigned long long excl; // kept words in all lower tiles
    uint32_t slot[kSlots];   // kept-word counts of the warp-vector slots
};

template <class Op>
__global__ void __launch_bounds__(kThreads, 2) irregular_kernel(const IrregParams p) {
    extern __shared__ __align__(128) uint32_t smem[];
    __shared__ __align__(8) uint64_t bar_full[kStages], bar_counted[kStages], bar_resolved[kStages],
        bar_empty[kStages];
    __shared__ StageMeta meta[kStages];
    __shared__ uint32_t s_epoch;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&bar_full[s], 1);
            mbar_init(&bar_counted[s], 1);
            mbar_init(&bar_resolved[s], 1);
            mbar_init(&bar_empty[s], kConsumerWarps);
        }
        mbar_fence_init();
    }
    __syncthreads();

    if (warp == 0) {
        // ------------------------------------------------ producer warp
        bool has_hprev = false;
        uint32_t hprev = 0;
        if (Op::kUnique) has_hprev = halo_prev(p, hprev);
        for (uint32_t k = 0;; ++k) {
            const int s = k % kStages;
            const uint32_t use = k / kStages;
            uint32_t* stage = smem + s * kStageWords;
            mbar_wait(&bar_empty[s], (use & 1) ^ 1);  // consumers released tile k - kStages
            uint32_t t = 0, epoch = 0;
            if (lane == 0) {
                draw_ticket(p.ctrl, p.draws, t, epoch);
                if (k == 0) s_epoch = epoch;
            }
            t = __shfl_sync(kFull, t, 0);
            epoch = __shfl_sync(kFull, epoch, 0);
            if (t >= p.ntiles) {  // one failed draw per CTA ends its work
                if (lane == 0) {
                    meta[s].tile = kNoTile;
                    mbar_arrive(&bar_counted[s]);
                }
                break;
            }
            const uint64_t tb = uint64_t(t) * kT;
            if (lane == 0) {
                debug_delay(t, 0);
                uint64_t end = tb + kT < p.hi ? tb + kT : p.hi;
                end = (end + 3) & ~3ull;  // may read <= 12 bytes past the array end (same 16 B chunk)
                const uint64_t beg = (Op::kUnique && t > 0) ? tb - 4 : tb;
                const uint32_t bytes = uint32_t(end - beg) * 4u;
                fence_proxy_async_smem();
                mbar_arrive_expect_tx(&bar_full[s], bytes);
                bulk_g2s(stage + kPre - (tb - beg), p.abase + beg, bytes, &bar_full[s]);
            }
            mbar_wait(&bar_full[s], use & 1);

            // a3 + a4: the tile aggregate.  Lane l counts words 4*(32j + l) + [0, 4),
            // j < T/128, then one warp reduction.
            uint32_t c = 0;
            if (tb >= p.lo && tb + kT <= p.hi) {
#pragma unroll 8
                for (int j = 0; j < kT / 128; ++j) {
                    const int x = 4 * (32 * j + lane);
                    const u32x4 q = *reinterpret_cast<const u32x4*>(stage + kPre + x);
                    if constexpr (Op::kUnique) {
                        const uint32_t pw = stage[kPre + x - 1];
                        c += (q.x != pw) + (q.y != q.x) + (q.z != q.y) + (q.w != q.z);
                    } else {
                        c += Op::keep(q.x, p.value) + Op::keep(q.y, p.value) + Op::keep(q.z, p.value) +
                             Op::keep(q.w, p.value);
                    }
                }
                if (Op::kUnique && tb == p.lo && lane == 0) {  // the array's first word (R18)
                    const uint32_t w0 = stage[kPre];
                    c += (!has_hprev || w0 != hprev) - (w0 != stage[kPre - 1]);
                }
            } else {  // the first (misaligned) or last (ragged) tile
                for (int j = 0; j < kT / 128; ++j) {
                    const int x = 4 * (32 * j + lane);
                    const u32x4 q = *reinterpret_cast<const u32x4*>(stage + kPre + x);
                    c += __popc(keep_mask<Op>(p, stage, tb, false, x, q, has_hprev, hprev));
                }
            }
            const uint32_t total = __reduce_add_sync(kFull, c);
            __syncwarp();
            if (lane == 0) {
                meta[s].tile = t;
                meta[s].total = total;
                debug_delay(t, 1);
                // a5a: publish the aggregate now -- it depends on nothing else.
                st_release_gpu(p.status + t, make_status(t == 0 ? kStateIncl : kStateAgg, epoch, total));
                mbar_arrive(&bar_counted[s]);
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------ resolver warp
        for (uint32_t k = 0;; ++k) {
            const int s = k % kStages;
            const uint32_t use = k / kStages;
            mbar_wait(&bar_counted[s], use & 1);
            const uint32_t t = meta[s].tile;
            if (t == kNoTile) {
                if (lane == 0) mbar_arrive(&bar_resolved[s]);
                break;
            }
            const uint32_t epoch = s_epoch;
            const uint32_t total = meta[s].total;
            if (lane == 0) debug_delay(t, 2);
            __syncwarp();
            const uint64_t excl = t > 0 ? lookback(p.status, t, epoch, lane) : 0ull;
            if (lane == 0) {
                if (t > 0) st_release_gpu(p.status + t, make_status(kStateIncl, epoch, excl + total));
                meta[s].excl = excl;
                if (t == p.ntiles - 1 && p.d_out_n) *p.d_out_n = excl + total;
                mbar_arrive(&bar_resolved[s]);
            }
        }
    } else {
        // ------------------------------------------------ consumer warps
        const int cw = warp - 2, ct = tid - 64;
        const uint32_t lt = lanemask_lt();
        bool has_hprev = false;
        uint32_t hprev = 0;
        if (Op::kUnique) has_hprev = halo_prev(p, hprev);
        for (uint32_t k = 0;; ++k) {
            const int s = k % kStages;
            const uint32_t use = k / kStages;
            uint32_t* stage = smem + s * kStageWords;
            mbar_wait(&bar_resolved[s], use & 1);
            const uint32_t t = meta[s].tile;
            if (t == kNoTile) break;
            const uint64_t tb = uint64_t(t) * kT;
            const bool full = tb >= p.lo && tb + kT <= p.hi;

            // a6: words -> registers, keep masks, in-warp exclusive ranks and the
            // count of every warp-vector slot (i, warp).
            uint32_t v[kVec][4];
            uint32_t masks = 0;                 // 4 bits per vector
            uint32_t lane_pre[kVec / 4] = {};   // 8 bits per vector (< 128)
#pragma unroll
            for (int i = 0; i < kVec; ++i) {
                const int x = 4 * (i * kCT + ct);
                const u32x4 q = *reinterpret_cast<const u32x4*>(stage + kPre + x);
                v[i][0] = q.x; v[i][1] = q.y; v[i][2] = q.z; v[i][3] = q.w;
                const uint32_t m = keep_mask<Op>(p, stage, tb, full, x, q, has_hprev, hprev);
                masks |= m << (4 * i);
                const uint32_t c = __popc(m);
                const uint32_t b0 = __ballot_sync(kFull, c & 1u);
                const uint32_t b1 = __ballot_sync(kFull, c & 2u);
                const uint32_t b2 = __ballot_sync(kFull, c & 4u);
                lane_pre[i / 4] |= (__popc(b0 & lt) + 2u * __popc(b1 & lt) + 4u * __popc(b2 & lt))
                                   << (8 * (i % 4));
                if (lane == 0) meta[s].slot[i * kConsumerWarps + cw] = __popc(b0) + 2u * __popc(b1) + 4u * __popc(b2);
            }
            named_bar_sync(1, kCT);  // slot counts written; every consumer holds its words

            // Exclusive scan of the 64 slot counts in input order, redundantly in
            // every warp (lane l holds slots l and l + 32).
            uint32_t ca = meta[s].slot[lane], cb = meta[s].slot[lane + 32];
            uint32_t ia = ca, ib = cb;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t ya = __shfl_up_sync(kFull, ia, o);
                const uint32_t yb = __shfl_up_sync(kFull, ib, o);
                if (lane >= o) {
                    ia += ya;
                    ib += yb;
                }
            }
            const uint32_t tot_a = __shfl_sync(kFull, ia, 31);
            const uint32_t ea = ia - ca, eb = tot_a + ib - cb;  // exclusive offsets of slots l, l+32

            // a7: scatter at the output's 16-byte phase, then aligned stores.
            const uint32_t A = meta[s].total;
            const uint64_t s0 = p.lo + meta[s].excl;
            uint32_t* out = stage + kPre + uint32_t(s0 & 3);
#pragma unroll
            for (int i = 0; i < kVec; ++i) {
                const int slot = i * kConsumerWarps + cw;  // warp-uniform
                const uint32_t base = __shfl_sync(kFull, slot < 32 ? ea : eb, slot & 31);
                uint32_t r = base + ((lane_pre[i / 4] >> (8 * (i % 4))) & 0xFFu);
                const uint32_t m = masks >> (4 * i);
#pragma unroll
                for (int kk = 0; kk < 4; ++kk)
                    if (m >> kk & 1u) out[r++] = v[i][kk];
            }
            named_bar_sync(1, kCT);  // compacted tile complete
            if (ct == 0) debug_delay(t, 3);
            const uint64_t s1 = s0 + A;
            const uint64_t c0 = s0 & ~3ull;
            const uint32_t nchunks = A ? uint32_t((s1 - c0 + 3) >> 2) : 0u;
#pragma unroll
            for (int it = 0; it < kVec + 1; ++it) {
                const uint32_t c = uint32_t(it * kCT + ct);
                if (c >= nchunks) break;
                const uint64_t g = c0 + 4ull * c;
                const u32x4 q = *reinterpret_cast<const u32x4*>(stage + kPre + 4 * c);
                if (g >= s0 && g + 4 <= s1) {
                    stg_stream_v4(p.abase + g, q.x, q.y, q.z, q.w);
                } else {
                    const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk)
                        if (g + kk >= s0 && g + kk < s1) stg_stream(p.abase + g + kk, w[kk]);
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&bar_empty[s]);  // this warp is done with the stage
        }
    }
}

struct LaunchCache {
    int dev = -1, sms = 0, per_sm = 0;
};

template <class Op>
cudaError_t launch_op(IrregParams p, cudaStream_t s) {
    static thread_local LaunchCache lc;
    auto kern = irregular_kernel<Op>;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (lc.dev != dev) {
        if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kSmem))) !=
            cudaSuccess)
            return e;
        if ((e = cudaDeviceGetAttribute(&lc.sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess)
            return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&lc.per_sm, kern, kThreads, kSmem)) !=
            cudaSuccess)
            return e;
        if (lc.per_sm < 1) lc.per_sm = 1;
        lc.dev = dev;
    }
    uint64_t grid = uint64_t(lc.sms) * lc.per_sm;
    if (grid > p.ntiles) grid = p.ntiles;
    p.draws = p.ntiles + uint32_t(grid);
    kern<<<uint32_t(grid), kThreads, kSmem, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

size_t irregular_tiles(const IrregArgs& a) {
    const uint64_t lo = (reinterpret_cast<uintptr_t>(a.ptr) >> 2) & 3u;
    return size_t((lo + a.n + kT - 1) / kT);
}

cudaError_t launch_irregular(const IrregArgs& a, Workspace& ws, cudaStream_t s) {
    IrregParams p{};
    const uint64_t lo = (reinterpret_cast<uintptr_t>(a.ptr) >> 2) & 3u;
    p.abase = a.ptr - lo;
    p.lo = lo;
    p.hi = lo + a.n;
    p.status = ws.status;
    p.ctrl = ws.ctrl;
    p.d_out_n = a.d_out_n;
    p.halo = a.halo;
    p.halo_len = uint32_t(a.halo_len);
    p.ntiles = uint32_t(irregular_tiles(a));
    p.value = a.value;
    count_launch();
    switch (a.op) {
    case IrregOp::Compact: return launch_op<OpCompact>(p, s);
    case IrregOp::Unique: return launch_op<OpUnique>(p, s);
    case IrregOp::Select:
        switch (a.predicate) {
        case 0: return launch_op<OpSelect<0>>(p, s);
        case 1: return launch_op<OpSelect<1>>(p, s);
        case 2: return launch_op<OpSelect<2>>(p, s);
        case 3: return launch_op<OpSelect<3>>(p, s);
        case 4: return launch_op<OpSelect<4>>(p, s);
        case 5: return launch_op<OpSelect<5>>(p, s);
        case 6: return launch_op<OpSelect<6>>(p, s);
        default: return cudaErrorInvalidValue;
        }
    }
    return cudaErrorInvalidValue;
}

}  // namespace ds
