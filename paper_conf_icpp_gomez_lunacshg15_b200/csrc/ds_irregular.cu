// ds_irregular.cu -- irregular Data Sliding on sm_100a: in-place, stable
// stream compaction, select and unique (Algorithm 2, P:168-190;
// §III-B; primitives §IV-B/C P:230-282).
//
// One CTA = one input tile of T = THREADS*ITEMS words, in dynamic-ticket
// order (Fig. 4).  Per tile:
//   a1 ticket                      -> draw_ticket()          (Fig. 4)
//   a2 load stage (registers)      -> 128-bit striped loads  (Alg. 2 L1-11)
//   a3 predicate / unique stencil  -> shfl_up + smem + one global boundary
//                                     read
//   a4 block reduce                -> ballot/popc + 1-warp scan ("Reduction",
//                                     P:182; before the sync)
//   a5 publish + resolve prefix    -> AGG status (release), decoupled look-back
//                                     over 32 predecessors, INCL status; this
//                                     replaces the serial flag chain of Fig. 7
//                                     (the chain is latency-bound
//                                     on B200)
//   a6 block scan                  -> rank of every kept word in input order
//                                     ("binary prefix sum")
//   a7 store stage                 -> smem compaction, 128-bit aligned stores
//                                     of [excl, excl+A), scalar head/tail
//   a8 finalise                    -> last tile writes out_n
//
// In-place safety: a tile stores only after the look-back saw AGG/INCL for
// every lower tile; statuses are published after the tile's loads; outputs
// of tile t lie in [0, (t+1)T) so no lower tile writes into a higher tile's
// input.  Deadlock freedom: waits only target lower tickets.
#include "ds_device.cuh"
#include "ds_internal.h"

namespace ds {
namespace {

constexpr unsigned kFull = 0xffffffffu;

struct IrregParams {
    uint32_t* abase;  // 16-byte-aligned base (ptr - lo)
    uint64_t lo, hi;  // valid virtual word range [lo, hi)
    uint64_t* status;
    uint64_t* ctrl;
    uint64_t* d_out_n;
    const uint64_t* halo;
    uint32_t halo_len;
    uint32_t ntiles;
    uint32_t value;  // compact: remove value; select: predicate parameter
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

// a5: decoupled look-back by one warp.  Returns the exclusive prefix
// (number of kept words in all tiles < tile).  Waits only for the lanes up
// to the nearest INCL predecessor.  Ends with one acquire fence per lane and
// a __syncwarp so lane 0's later release is cumulative over all lanes.
__device__ __forceinline__ uint64_t lookback(const uint64_t* __restrict__ status, uint32_t tile,
                                             uint32_t epoch, int lane) {
    uint64_t excl = 0;
    int64_t base = int64_t(tile) - 1;
    while (true) {
        const int64_t idx = base - lane;
        uint64_t s = make_status(kStateIncl, epoch, 0);  // virtual INCL(0) before tile 0
        bool ok = true;
        if (idx >= 0) {
            s = ld_relaxed_gpu(status + idx);
            ok = status_current(s, epoch);
        }
        uint32_t ns = 8;
        while (true) {
            const uint32_t incl = __ballot_sync(kFull, ok && status_state(s) == kStateIncl);
            const uint32_t need = incl ? ((incl & (0u - incl)) << 1) - 1u : kFull;
            const uint32_t bad = __ballot_sync(kFull, !ok);
            if ((bad & need) == 0) break;
            __nanosleep(ns);
            ns = ns < 256 ? ns * 2 : 256;
            if (!ok) {
                s = ld_relaxed_gpu(status + idx);
                ok = status_current(s, epoch);
            }
        }
        const uint32_t incl = __ballot_sync(kFull, ok && status_state(s) == kStateIncl);
        if (incl) {
            const int L = __ffs(incl) - 1;
            const uint32_t agg = lane < L ? uint32_t(status_count(s)) : 0u;
            const uint64_t inc = __shfl_sync(kFull, status_count(s), L);
            excl += uint64_t(__reduce_add_sync(kFull, agg)) + inc;
            break;
        }
        excl += __reduce_add_sync(kFull, uint32_t(status_count(s)));
        base -= 32;
    }
    fence_acq_rel_gpu();
    __syncwarp();
    return excl;
}

template <int THREADS, int ITEMS, class Op>
__global__ void __launch_bounds__(THREADS) irregular_kernel(const IrregParams p) {
    static_assert(ITEMS % 4 == 0 && THREADS % 32 == 0, "tile shape");
    constexpr int VEC = ITEMS / 4;
    constexpr int WARPS = THREADS / 32;
    constexpr int T = THREADS * ITEMS;
    constexpr int SLOTS = VEC * WARPS;
    constexpr int SPL = (SLOTS + 31) / 32;

    __shared__ uint32_t s_tile, s_epoch, s_total;
    __shared__ unsigned long long s_excl;
    __shared__ uint32_t s_slot[SPL * 32];
    __shared__ uint32_t s_last[Op::kUnique ? SLOTS : 1];
    __shared__ alignas(16) uint32_t s_buf[T];

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

    if (tid == 0) {  // a1
        uint32_t t, e;
        draw_ticket(p.ctrl, p.ntiles, t, e);
        s_tile = t;
        s_epoch = e;
        debug_delay(t, 0);
    }
    __syncthreads();
    const uint32_t tile = s_tile, epoch = s_epoch;
    const uint64_t tb = uint64_t(tile) * T;
    const bool full = tb >= p.lo && tb + T <= p.hi;

    // a2: load stage.  Vector i of thread tid covers words tb + 4*(i*THREADS+tid) + [0,4).
    uint32_t v[VEC][4];
#pragma unroll
    for (int i = 0; i < VEC; ++i) {
        const uint64_t e0 = tb + 4ull * uint64_t(i * THREADS + tid);
        if (full || (e0 >= p.lo && e0 + 4 <= p.hi)) {
            const u32x4 q = ldg_stream_v4(p.abase + e0);
            v[i][0] = q.x; v[i][1] = q.y; v[i][2] = q.z; v[i][3] = q.w;
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint64_t e = e0 + k;
                v[i][k] = (e >= p.lo && e < p.hi) ? ldg_stream(p.abase + e) : 0u;
            }
        }
    }

    // Unique: predecessor of the tile's first word ("on the boundaries
    // we directly access global memory"), or the shard halo (R18) for the
    // array's first word.  Only thread 0 needs it.
    uint32_t first_prev = 0;
    bool first_has_prev = false;
    if constexpr (Op::kUnique) {
        if (tid == 0) {
            if (tb > p.lo) {
                first_prev = ldg_stream(p.abase + tb - 1);
                first_has_prev = true;
            } else {
                for (uint32_t h = p.halo_len; h-- > 0;) {
                    const uint64_t ent = p.halo[h];
                    if (ent >> 32) {
                        first_prev = uint32_t(ent);
                        first_has_prev = true;
                        break;
                    }
                }
            }
        }
        if (lane == 31) {
#pragma unroll
            for (int i = 0; i < VEC; ++i) s_last[i * WARPS + warp] = v[i][3];
        }
        __syncthreads();
    }

    // a3 + a4: keep masks, per-warp-vector counts via ballot bit slices.
    uint32_t mask[VEC], lane_pre[VEC];
    const uint32_t lt = lanemask_lt();
#pragma unroll
    for (int i = 0; i < VEC; ++i) {
        const uint64_t e0 = tb + 4ull * uint64_t(i * THREADS + tid);
        uint32_t m = 0;
        if constexpr (Op::kUnique) {
            uint32_t pr = __shfl_up_sync(kFull, v[i][3], 1);
            if (lane == 0) {
                if (warp > 0) pr = s_last[i * WARPS + warp - 1];
                else if (i > 0) pr = s_last[(i - 1) * WARPS + WARPS - 1];
                else pr = first_prev;
            }
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint64_t e = e0 + k;
                const uint32_t prev = k ? v[i][k - 1] : pr;
                bool kp;
                if (e == p.lo) kp = !first_has_prev || v[i][k] != first_prev;
                else kp = v[i][k] != prev;
                if ((full || (e >= p.lo && e < p.hi)) && kp) m |= 1u << k;
            }
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint64_t e = e0 + k;
                if ((full || (e >= p.lo && e < p.hi)) && Op::keep(v[i][k], p.value)) m |= 1u << k;
            }
        }
        mask[i] = m;
        const uint32_t c = __popc(m);
        const uint32_t b0 = __ballot_sync(kFull, c & 1u);
        const uint32_t b1 = __ballot_sync(kFull, c & 2u);
        const uint32_t b2 = __ballot_sync(kFull, c & 4u);
        lane_pre[i] = __popc(b0 & lt) + 2u * __popc(b1 & lt) + 4u * __popc(b2 & lt);
        if (lane == 0) s_slot[i * WARPS + warp] = __popc(b0) + 2u * __popc(b1) + 4u * __popc(b2);
    }
    __syncthreads();  // all loads of this tile are performed (values consumed above)

    // a4/a6: one warp scans the per-(vector, warp) totals in input order and
    // publishes the tile aggregate as early as possible.
    uint32_t total = 0;
    if (warp == 0) {
        uint32_t vals[SPL], sum = 0;
#pragma unroll
        for (int j = 0; j < SPL; ++j) {
            const int idx = lane * SPL + j;
            vals[j] = idx < SLOTS ? s_slot[idx] : 0u;
            sum += vals[j];
        }
        uint32_t incl = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += y;
        }
        total = __shfl_sync(kFull, incl, 31);
        uint32_t run = incl - sum;
#pragma unroll
        for (int j = 0; j < SPL; ++j) {
            const int idx = lane * SPL + j;
            if (idx < SLOTS) s_slot[idx] = run;
            run += vals[j];
        }
        if (lane == 0) {
            s_total = total;
            debug_delay(tile, 1);
            st_release_gpu(p.status + tile,
                           make_status(tile == 0 ? kStateIncl : kStateAgg, epoch, total));
        }
    }
    __syncthreads();

    // a6: scatter kept words to their in-tile rank (independent of excl, so
    // it overlaps warp 0's look-back).
#pragma unroll
    for (int i = 0; i < VEC; ++i) {
        uint32_t r = s_slot[i * WARPS + warp] + lane_pre[i];
#pragma unroll
        for (int k = 0; k < 4; ++k)
            if (mask[i] >> k & 1u) s_buf[r++] = v[i][k];
    }

    // a5 + a8
    if (warp == 0) {
        if (lane == 0) debug_delay(tile, 2);
        __syncwarp();
        const uint64_t excl = tile > 0 ? lookback(p.status, tile, epoch, lane) : 0ull;
        if (lane == 0) {
            if (tile > 0) st_release_gpu(p.status + tile, make_status(kStateIncl, epoch, excl + total));
            s_excl = excl;
            if (tile == p.ntiles - 1 && p.d_out_n) *p.d_out_n = excl + total;
        }
    }
    __syncthreads();

    // a7: store stage -- [excl, excl + A) in 16-byte chunks; only whole
    // chunks inside the range use STG.128, the (at most two) partial chunks
    // are written word by word so no word outside the range is touched.
    const uint32_t A = s_total;
    if (A == 0) return;
    if (tid == 0) debug_delay(tile, 3);
    const uint64_t s0 = p.lo + s_excl;
    const uint64_t s1 = s0 + A;
    const uint64_t c0 = s0 & ~3ull;
    const uint32_t nchunks = uint32_t((s1 - c0 + 3) >> 2);
#pragma unroll
    for (int it = 0; it < VEC + 1; ++it) {
        const uint32_t c = uint32_t(it * THREADS + tid);
        if (c >= nchunks) break;
        const uint64_t g = c0 + 4ull * c;
        if (g >= s0 && g + 4 <= s1) {
            const uint32_t o = uint32_t(g - s0);
            stg_stream_v4(p.abase + g, s_buf[o], s_buf[o + 1], s_buf[o + 2], s_buf[o + 3]);
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint64_t e = g + k;
                if (e >= s0 && e < s1) stg_stream(p.abase + e, s_buf[e - s0]);
            }
        }
    }
}

// Tile shape: 256 threads x 16 words = 16 KB per CTA (the paper's WG 256 x
// coarsening factor 16), tuned on B200 in DESIGN.md §7.
constexpr int kThreads = 256;
constexpr int kItems = 16;
constexpr int kTile = kThreads * kItems;

template <class Op>
cudaError_t launch_op(const IrregParams& p, cudaStream_t s) {
    irregular_kernel<kThreads, kItems, Op><<<p.ntiles, kThreads, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

size_t irregular_tiles(const IrregArgs& a) {
    const uint64_t lo = (reinterpret_cast<uintptr_t>(a.ptr) >> 2) & 3u;
    return size_t((lo + a.n + kTile - 1) / kTile);
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
