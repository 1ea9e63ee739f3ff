// ds_irregular.cu -- irregular Data Sliding on sm_100a: in-place, stable
// stream compaction, select and unique (Algorithm 2, P:168-190;
// §III-B; primitives §IV-B/C P:230-282).
//
// One persistent, warp-specialised CTA per SM walks input tiles of
// T = 8192 words in dynamic-ticket order (Fig. 4) through a 6-stage ring of
// shared-memory tiles.  Each role works on a different tile at a time:
//
//   producer warp    a1 draws the next ticket as soon as a stage is free and
//                    a2 loads the tile (plus, for unique, the 16 bytes before
//                       it) with one TMA bulk copy (Alg. 2 lines 1-11; P:84
//                       "on-chip memory")
//  16 ranker warps   a3 keep flags (predicate / unique stencil), one
//                       ballot per 32-word chunk (lane l holds word 32c + l)
//                    a4 the tile aggregate ("Reduction") -- published
//                       as AGG at once
//                    a6 rank of every kept word in input order ("binary
//                       prefix sum": popc of the chunk ballot
//                       below the lane + a scan of the 16 warp totals); the
//                       kept words are compacted in place, 32 consecutive
//                       words per store
//   6 resolver warps a5 (one per stage) decoupled look-back over 32
//                       predecessors per round trip, started as soon as the
//                       ticket is drawn (it needs no data), then INCL; the last
//                       tile writes out_n (a8).  This replaces the serial flag
//                       chain of Fig. 7, which is latency-bound on B200
//
//   5 storer warps   a7 re-phase the compacted words in shared memory to the
//                       destination's 16-byte phase, one TMA bulk store of
//                       [excl, excl + A) (scalar head/tail), then free the
//                       stage once the bulk engine has read it
//
// A drawn tile's AGG depends only on its own load and ranking, never on the
// resolution of earlier tiles.  In-place safety:
// AGG/INCL are published only after the tile's copy completed; stores happen
// only after the look-back saw AGG/INCL of every lower tile; outputs of tile t
// lie in [0, (t+1)T), so no lower tile writes into a higher tile's input.
// Deadlock freedom: look-backs wait only for lower (already drawn) tiles, and
// a drawn tile reaches AGG without waiting on any other tile.
#include <type_traits>

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
    uint32_t value_hi;  // 8-byte elements: high word of the value / parameter
    uint32_t wshift;    // out_n = words >> wshift (1 for 8-byte elements)
    uint64_t* trace;  // diagnostics: per-tile events, or null
    uint32_t* tbase;  // 16-byte-aligned base of the true/kept output (== abase in place)
    uint64_t tlo;     // its word offset (output word j lives at tbase[tlo + j])
    uint32_t* fbase;  // same for the false words (partition), or null
    uint64_t flo;
};

// ---- predicates (a3) ----------------------------------------------------
// kWide: the elements are 8 bytes (two consecutive words, the low word first);
// both words of an element get the element's keep flag, so ranks, prefixes
// and stores stay in words and every kept element moves as a pair.
struct OpCompact {  // remove words equal to a value
    static constexpr bool kUnique = false, kWide = false;
    __device__ static bool keep(uint32_t w, uint32_t v) { return w != v; }
};
template <int P>
struct OpSelect {  // keep predicate-true words (R14); ids = ds_predicate
    static constexpr bool kUnique = false, kWide = false;
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
    static constexpr bool kUnique = true, kWide = false;
    __device__ static bool keep(uint32_t, uint32_t) { return true; }
};
// 8-byte elements: same primitives on int64 / float64 values.
struct OpCompact64 {
    static constexpr bool kUnique = false, kWide = true;
    __device__ static bool keep2(uint64_t e, uint64_t v) { return e != v; }
};
template <int P>
struct OpSelect64 {  // ds_predicate ids with the element type widened: I32 -> int64, F32 -> double
    static constexpr bool kUnique = false, kWide = true;
    __device__ static bool keep2(uint64_t e, uint64_t param) {
        if constexpr (P == 0) return e != 0ull;
        else if constexpr (P == 1) return int64_t(e) > int64_t(param);
        else if constexpr (P == 2) return !(int64_t(e) > int64_t(param));
        else if constexpr (P == 3) return __longlong_as_double(int64_t(e)) > __longlong_as_double(int64_t(param));
        else if constexpr (P == 4) return !(__longlong_as_double(int64_t(e)) > __longlong_as_double(int64_t(param)));
        else if constexpr (P == 5) return (e & 1ull) == 0ull;
        else return (e & 1ull) != 0ull;
    }
};
struct OpUnique64 {
    static constexpr bool kUnique = true, kWide = true;
};

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// ---- CTA shape ----------------------------------------------------------
#ifndef DS_IRR_RANK_WARPS
#define DS_IRR_RANK_WARPS 16
#endif
#ifndef DS_IRR_IN_STAGES
#define DS_IRR_IN_STAGES 6
#endif
#ifndef DS_IRR_SLOTS
#define DS_IRR_SLOTS 12
#endif
#ifndef DS_IRR_RESOLVERS
#define DS_IRR_RESOLVERS 6
#endif
#ifndef DS_IRR_RANK_GROUPS
#define DS_IRR_RANK_GROUPS 1
#endif
#ifndef DS_IRR_TILE
#define DS_IRR_TILE 8192
#endif
constexpr int kRankWarps = DS_IRR_RANK_WARPS;
constexpr int kRankGroups = DS_IRR_RANK_GROUPS;   // ranker groups, each on its own tile
constexpr int kGroupWarps = kRankWarps / kRankGroups;
constexpr int kRT = 32 * kGroupWarps;     // threads of one ranker group
constexpr int kT = DS_IRR_TILE;           // words per tile (8192 = 32 KB)
constexpr int kSeg = kT / kGroupWarps;    // contiguous words ranked by one warp (1024)
constexpr int kChunks = kSeg / 32;        // 32-word chunks per warp segment (32)
static_assert(kRankWarps % kRankGroups == 0 && kT % (32 * kGroupWarps) == 0, "ranker shape");
static_assert(kChunks <= 32, "chunk masks are held one per lane");
static_assert(kRankGroups <= 2, "named barriers 1 and 3 serve the ranker groups");
constexpr int kInStages = DS_IRR_IN_STAGES;   // input tiles (TMA destination)
constexpr int kSlots = DS_IRR_SLOTS;          // tiles in flight per CTA (meta ring)
constexpr int kResolvers = DS_IRR_RESOLVERS;  // resolver r serves ring positions k = r mod kResolvers
#ifndef DS_IRR_STORE_WARPS
#define DS_IRR_STORE_WARPS 5
#endif
constexpr int kStoreWarps = DS_IRR_STORE_WARPS;
#ifndef DS_IRR_BULK_STORE
#define DS_IRR_BULK_STORE 1
#endif
constexpr bool kBulkStore = DS_IRR_BULK_STORE;  // a7 through TMA bulk stores (else 128-bit STG)
constexpr int kST = 32 * kStoreWarps;
constexpr int kWarpResolver0 = kRankWarps;
constexpr int kWarpStorer0 = kRankWarps + kResolvers;
constexpr int kWarpProducer = kWarpStorer0 + kStoreWarps;
constexpr int kThreads = 32 * (kWarpProducer + 1);
#ifndef DS_IRR_PRE
#define DS_IRR_PRE 32
#endif
// Words before the tile in a stage (unique's boundary word).  Stages, and the
// tile inside each stage, start on 128-byte boundaries, so a bulk copy fills
// whole 128-byte shared-memory lines and unique's copy (which starts kPre
// words early) keeps a 128-byte aligned global source.
constexpr int kPre = DS_IRR_PRE;
#ifndef DS_IRR_ALIGN
#define DS_IRR_ALIGN 32
#endif
constexpr int kAlignW = DS_IRR_ALIGN;    // stage alignment in words (32 = 128 bytes)
constexpr int kStageWords = (kT + kPre + 4 + kAlignW - 1) / kAlignW * kAlignW;
constexpr size_t kSmem = size_t(kInStages) * kStageWords * 4 + 128;  // + runtime alignment slack
static_assert(kPre % 4 == 0 && kPre >= 4, "boundary words keep 16-byte alignment");
static_assert(!DS_IRR_BULK_STORE || kStageWords >= kT + kPre + 8,
              "re-phase writes whole chunks up to 6 words past a segment");
static_assert(kThreads <= 1024, "CTA size");
static_assert(kSlots >= kInStages, "a slot per input stage at least");
static_assert(kSlots % kResolvers == 0, "a slot is always served by the same resolver");
// 227 KB dynamic + static per CTA (the static part -- barriers, slot metadata --
// is < 2.5 KB)
static_assert(kSmem <= 227 * 1024 - 2560, "shared memory");

struct SlotMeta {
    uint32_t tile;              // kNoTile: end of this CTA's work
    uint32_t prev_tile;         // this CTA's previous ticket (kNoTile: none)
    volatile uint32_t incl_tile;          // == tile once incl is valid (CTA-local chain)
    volatile unsigned long long incl;     // inclusive prefix of the tile
    uint32_t total;             // kept words in the tile
    unsigned long long excl;    // kept words in all lower tiles
    uint32_t wtot[kGroupWarps];  // kept words in each ranker warp's segment
};

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

// a5: decoupled look-back by one warp over 32 * kLB predecessors per round trip
// (kLB = 1: fewer status sectors per poll beat a wider window).
// Slot (m, lane) examines tile base - (32m + lane): every load instruction
// reads 32 consecutive status words.  Waits only for the tiles up to the
// nearest INCL predecessor.  Ends with one acquire fence per lane and a
// __syncwarp so lane 0's later release is cumulative over all lanes.
#ifndef DS_IRR_LB
#define DS_IRR_LB 1
#endif
constexpr int kLB = DS_IRR_LB;  // look-back slots per lane (kLBW * kLB tiles per round)
#ifndef DS_IRR_LBW
#define DS_IRR_LBW 32
#endif
constexpr int kLBW = DS_IRR_LBW;  // lanes that read statuses (window width per slot row)
static_assert(kLBW >= 1 && kLBW <= 32, "look-back lanes");
#ifndef DS_IRR_REFRESH
#define DS_IRR_REFRESH 1
#endif
#ifndef DS_IRR_POLL_MIN
#define DS_IRR_POLL_MIN 64
#endif
#ifndef DS_IRR_POLL_MAX
#define DS_IRR_POLL_MAX 512
#endif
constexpr int kRefreshRows = DS_IRR_REFRESH;        // AGG rows re-read while polling
constexpr uint32_t kPollMinNs = DS_IRR_POLL_MIN;   // first back-off
constexpr uint32_t kPollMaxNs = DS_IRR_POLL_MAX;   // back-off cap

// Timing experiments only (wrong or unsafe results): DS_DEBUG_BISECT bits
#ifndef DS_DEBUG_BISECT
#define DS_DEBUG_BISECT 0
#endif
constexpr bool DBG_NO_PFENCE = DS_DEBUG_BISECT & 1, DBG_NO_PUBLISH = DS_DEBUG_BISECT & 2,
               DBG_NO_BULKWAIT = DS_DEBUG_BISECT & 4, DBG_EARLY_FREE = DS_DEBUG_BISECT & 8,
               DBG_SKIP_RANK = DS_DEBUG_BISECT & 16, DBG_NO_RFENCE = DS_DEBUG_BISECT & 32;
#ifndef DS_IRR_LATE_LB
#define DS_IRR_LATE_LB 0
#endif
#ifndef DS_IRR_HELP
#define DS_IRR_HELP 0
#endif
constexpr bool kHelp = DS_IRR_HELP;  // publish INCL for the nearest 32 AGG predecessors
static_assert(!kHelp || kLBW == 32, "helper INCLs assume the 32-lane window");

__device__ __forceinline__ uint64_t lookback(uint64_t* __restrict__ status, uint32_t tile,
                                             uint32_t epoch, int lane, uint64_t* trace) {
    uint64_t excl = 0;
    uint32_t rounds = 0, polls = 0;
    int64_t base = int64_t(tile) - 1;
    uint64_t s0 = 0;     // the nearest 32 predecessors' statuses as the first round left them
    uint32_t L0 = 32u;   // lanes of that row the walk needed (up to the nearest INCL)
    while (true) {
        uint64_t s[kLB];
        uint32_t okm = 0;  // bit m: slot m holds a current status
        const bool act = lane < kLBW;  // lanes of the window (the rest read as empty, current)
#pragma unroll
        for (int m = 0; m < kLB; ++m) {
            const int64_t idx = base - (kLBW * m + lane);
            s[m] = !act ? 0ull : idx >= 0 ? ld_relaxed_gpu(status_ptr(status, idx)) : make_status(kStateIncl, epoch, 0);
        }
#pragma unroll
        for (int m = 0; m < kLB; ++m)
            if (!act || status_current(s[m], epoch)) okm |= 1u << m;
        if (rounds++ == 0 && lane == 0) trace_event(trace, tile, 10, globaltimer());
        uint32_t ns = kPollMinNs;
        uint32_t M, L;  // nearest INCL at slot M, lane L (M == kLB: none this round)
        while (true) {
            uint32_t inclm = 0;
#pragma unroll
            for (int m = 0; m < kLB; ++m)
                if ((okm >> m & 1u) && status_state(s[m]) == kStateIncl) inclm |= 1u << m;
            M = __reduce_min_sync(kFull, inclm ? uint32_t(__ffs(inclm) - 1) : uint32_t(kLB));
            L = M < kLB ? uint32_t(__ffs(__ballot_sync(kFull, inclm >> M & 1u)) - 1) : 32u;
            // needed: every slot before (M, L) in distance order, and (M, L)
            const uint32_t need = (M < kLB ? ((1u << M) - 1u) : ((1u << kLB) - 1u)) |
                                  (M < kLB && uint32_t(lane) <= L ? (1u << M) : 0u);
            if (!__any_sync(kFull, (okm & need) != need)) break;
            __nanosleep(ns);
            ns = ns < kPollMaxNs ? ns * 2 : kPollMaxNs;
            ++polls;
            // Re-read the needed slots that are still pending, and refresh the
            // nearest 32 predecessors even if they hold AGG: a nearer INCL ends the
            // walk sooner.  Farther AGG slots are not re-read (poll traffic hits
            // the same few L2 lines from every resolver).
#pragma unroll
            for (int m = 0; m < kLB; ++m) {
                const bool pending = !(okm >> m & 1u);
                const bool refresh = act && m < kRefreshRows && !pending && status_state(s[m]) != kStateIncl;
                if ((need >> m & 1u) && (pending || refresh)) {
                    const int64_t idx = base - (kLBW * m + lane);
                    if (idx >= 0) {
                        s[m] = ld_relaxed_gpu(status_ptr(status, idx));
                        okm = status_current(s[m], epoch) ? (okm | 1u << m) : (okm & ~(1u << m));
                    }
                }
            }
        }
        uint32_t agg = 0;
        uint64_t inc = 0;
#pragma unroll
        for (int m = 0; m < kLB; ++m) {
            if (uint32_t(m) < M || (uint32_t(m) == M && uint32_t(lane) < L)) agg += uint32_t(status_count(s[m]));
            if (uint32_t(m) == M && uint32_t(lane) == L) inc = status_count(s[m]);
        }
        excl += uint64_t(__reduce_add_sync(kFull, agg));
        if (rounds == 1) {
            s0 = s[0];
            L0 = M == 0 ? L : 32u;
        }
        if (M < kLB) {
            excl += __shfl_sync(kFull, inc, L);
            break;
        }
        base -= kLBW * kLB;
    }
    if (kHelp) {
        // The walk fixed the inclusive prefix of every tile it summed: for the
        // nearest predecessors t-1-l (l < L0, all AGG), incl = excl - (counts of
        // t-1 .. t-l).  Publishing them lets later look-backs stop sooner.  A
        // racing writer (the tile's own resolver, another helper) stores the
        // same word.
        const uint32_t c0 = uint32_t(lane) < L0 ? uint32_t(status_count(s0)) : 0u;
        uint32_t pre = c0;
#pragma unroll
        for (int sh = 1; sh < 32; sh <<= 1) {
            const uint32_t y = __shfl_up_sync(kFull, pre, sh);
            if (lane >= sh) pre += y;
        }
        pre -= c0;  // exclusive: counts of the lanes nearer than this one
        const int64_t idx = int64_t(tile) - 1 - lane;
        if (uint32_t(lane) < L0 && idx >= 0 && status_state(s0) == kStateAgg)
            publish_status(status_ptr(status, idx), make_status(kStateIncl, epoch, excl - pre));
    }
    if (lane == 0) {
        trace_event(trace, tile, 8, rounds);
        trace_event(trace, tile, 9, polls);
        trace_event(trace, tile, 11, globaltimer());
    }
    lookback_acquire();
    __syncwarp();
    if (lane == 0) trace_event(trace, tile, 12, globaltimer());
    return excl;
}

#ifndef DS_IRR_LOCAL_CHAIN
#define DS_IRR_LOCAL_CHAIN 0
#endif
constexpr bool kLocalChain = DS_IRR_LOCAL_CHAIN;
#ifndef DS_IRR_LW
#define DS_IRR_LW 8
#endif
constexpr int kLW = DS_IRR_LW;  // window slots per lane (32 * kLW tiles)

// a5, CTA-local chain: this CTA's previous tile tp < t resolves first (its
// resolver is in the same CTA), so t needs only the aggregates of the window
// (tp, t) -- about one tile per other SM -- plus incl(tp) from shared memory,
// or a nearer INCL inside the window.  One read of the window (<= 32*kLB
// tiles), then only its pending slots are re-read; no multi-round walk.
__device__ __forceinline__ uint64_t lookback_window(const uint64_t* __restrict__ status, uint32_t tile,
                                                    uint32_t tp, const SlotMeta* pm, uint32_t epoch,
                                                    int lane, uint64_t* trace) {
    const uint32_t W = tile - tp - 1;  // window tiles tile-1 .. tp+1
    const int64_t base = int64_t(tile) - 1;
    uint64_t s[kLW];
    uint32_t okm = 0;  // bit m: slot m current (or outside the window)
#pragma unroll
    for (int m = 0; m < kLW; ++m) {
        const uint32_t d = uint32_t(32 * m + lane);
        if (d < W) {
            s[m] = ld_relaxed_gpu(status_ptr(status, base - d));
            if (status_current(s[m], epoch)) okm |= 1u << m;
        } else {
            s[m] = 0;
            okm |= 1u << m;
        }
    }
    if (lane == 0) trace_event(trace, tile, 10, globaltimer());
    uint32_t ns = kPollMinNs, polls = 0;
    uint32_t M, L;
    bool local;
    while (true) {
        uint32_t inclm = 0;
#pragma unroll
        for (int m = 0; m < kLW; ++m)
            if (uint32_t(32 * m + lane) < W && (okm >> m & 1u) && status_state(s[m]) == kStateIncl) inclm |= 1u << m;
        M = __reduce_min_sync(kFull, inclm ? uint32_t(__ffs(inclm) - 1) : uint32_t(kLW));
        L = M < kLW ? uint32_t(__ffs(__ballot_sync(kFull, inclm >> M & 1u)) - 1) : 32u;
        const uint32_t need = (M < kLW ? ((1u << M) - 1u) : ((1u << kLW) - 1u)) |
                              (M < kLW && uint32_t(lane) <= L ? (1u << M) : 0u);
        const bool have = !__any_sync(kFull, (okm & need) != need);
        local = M == kLW && __shfl_sync(kFull, pm->incl_tile, 0) == tp;
        if (have && (M < kLW || local)) break;
        __nanosleep(ns);
        ns = ns < kPollMaxNs ? ns * 2 : kPollMaxNs;
        ++polls;
#pragma unroll
        for (int m = 0; m < kLW; ++m) {
            const bool pending = !(okm >> m & 1u);
            const bool refresh = m < kRefreshRows && !pending && status_state(s[m]) != kStateIncl;
            if ((need >> m & 1u) && (pending || (refresh && !local))) {
                const int64_t idx = base - (32 * m + lane);
                if (uint32_t(32 * m + lane) < W) {
                    s[m] = ld_relaxed_gpu(status_ptr(status, idx));
                    okm = status_current(s[m], epoch) ? (okm | 1u << m) : (okm & ~(1u << m));
                }
            }
        }
    }
    uint32_t agg = 0;
    uint64_t inc = 0;
#pragma unroll
    for (int m = 0; m < kLW; ++m) {
        const bool inw = uint32_t(32 * m + lane) < W;
        if (inw && (uint32_t(m) < M || (uint32_t(m) == M && uint32_t(lane) < L))) agg += uint32_t(status_count(s[m]));
        if (uint32_t(m) == M && uint32_t(lane) == L) inc = status_count(s[m]);
    }
    uint64_t excl = uint64_t(__reduce_add_sync(kFull, agg));
    __threadfence_block();  // incl was written before incl_tile
    excl += M < kLW ? __shfl_sync(kFull, inc, L) : pm->incl;
    if (lane == 0) {
        trace_event(trace, tile, 8, M < kLW ? 1 : 0);
        trace_event(trace, tile, 9, polls);
        trace_event(trace, tile, 11, globaltimer());
    }
    lookback_acquire();
    __syncwarp();
    if (lane == 0) trace_event(trace, tile, 12, globaltimer());
    return excl;
}

// a7 helper: write the `cnt` words stage[src_off, src_off + cnt) to the
// output words base[d0, d0 + cnt) (virtual indices; base is 16-byte aligned).
// Destination chunks of 4 aligned words are read as two aligned shared
// vectors and funnel-shifted (the phase is uniform over the segment); whole
// chunks use one STG.128, the head and tail chunks are written word by word
// so no word outside the segment is touched.  kSTT threads, 4 chunks per
// iteration for ILP.
template <int kSTT>
__device__ __forceinline__ void store_segment(uint32_t* base, uint64_t d0, uint32_t cnt,
                                              const uint32_t* stage, int32_t src_off, int st) {
    if (cnt == 0) return;
    const uint64_t d1 = d0 + cnt;
    const uint64_t c0 = d0 & ~3ull;
    const int32_t bidx = src_off - int32_t(d0 & 3);  // stage index of chunk 0's first word
    const uint32_t ph = uint32_t(bidx) & 3u;
    const uint32_t* sv = stage + (bidx & ~3);
    const uint32_t nchunks = uint32_t((d1 - c0 + 3) >> 2);
    constexpr int kU = 4;
    for (uint32_t c0i = st; c0i < nchunks; c0i += kU * kSTT) {
        uint32_t w[kU][4];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const uint32_t c = c0i + u * kSTT;
            if (c < nchunks) {
                const u32x4 lo = *reinterpret_cast<const u32x4*>(sv + 4 * c);
                const u32x4 hi = ph ? *reinterpret_cast<const u32x4*>(sv + 4 * c + 4) : lo;
                switch (ph) {  // warp-uniform
                case 0: w[u][0] = lo.x; w[u][1] = lo.y; w[u][2] = lo.z; w[u][3] = lo.w; break;
                case 1: w[u][0] = lo.y; w[u][1] = lo.z; w[u][2] = lo.w; w[u][3] = hi.x; break;
                case 2: w[u][0] = lo.z; w[u][1] = lo.w; w[u][2] = hi.x; w[u][3] = hi.y; break;
                default: w[u][0] = lo.w; w[u][1] = hi.x; w[u][2] = hi.y; w[u][3] = hi.z; break;
                }
            }
        }
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const uint32_t c = c0i + u * kSTT;
            if (c >= nchunks) break;
            const uint64_t g = c0 + 4ull * c;
            if (g >= d0 && g + 4 <= d1) {
                stg_stream_v4(base + g, w[u][0], w[u][1], w[u][2], w[u][3]);
            } else {
#pragma unroll
                for (int kk = 0; kk < 4; ++kk)
                    if (g + kk >= d0 && g + kk < d1) stg_stream(base + g + kk, w[u][kk]);
            }
        }
    }
}

// a7 helper: move the cnt words seg[0, cnt) to seg[ph, ph + cnt) in shared
// memory (ph = 1..3; seg 16-byte aligned with >= 4 readable words before it
// and >= 4 writable words after the segment).  Destination chunk c (words
// [4c, 4c+4)) takes source words [4c-ph, 4c+4-ph): two aligned vector loads.
// Writing chunk c destroys sources of chunk c+1 only, so the chunks go in
// descending rounds, each reading everything before writing.
template <int kSTT>
__device__ __forceinline__ void rephase(uint32_t* seg, uint32_t cnt, uint32_t ph, int st) {
    constexpr int kU = 4;
    const int32_t nchunks = int32_t((cnt + ph + 3) >> 2);
    for (int32_t hi = nchunks; hi > 0; hi -= kU * kSTT) {
        const int32_t lo = hi - kU * kSTT;
        u32x4 w[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int32_t c = lo + u * kSTT + st;
            if (c >= 0 && c < hi) {
                const u32x4 a = *reinterpret_cast<const u32x4*>(seg + 4 * c - 4);
                const u32x4 b = *reinterpret_cast<const u32x4*>(seg + 4 * c);
                switch (ph) {  // uniform
                case 1: w[u] = u32x4{a.w, b.x, b.y, b.z}; break;
                case 2: w[u] = u32x4{a.z, a.w, b.x, b.y}; break;
                default: w[u] = u32x4{a.y, a.z, a.w, b.x}; break;
                }
            }
        }
        named_bar_sync(2, kSTT);
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int32_t c = lo + u * kSTT + st;
            if (c >= 0 && c < hi) *reinterpret_cast<u32x4*>(seg + 4 * c) = w[u];
        }
        named_bar_sync(2, kSTT);
    }
}


// mbarrier wait that also returns (false) once the CTA's work is known to
// end before ring position k (the resolvers take alternate positions, so the
// one not holding the end marker is released this way).
// Suspend-time hint of those waits: it bounds how long a warp parked on a
// position past the end keeps the CTA (and so the launch) alive.
#ifndef DS_IRR_END_POLL_NS
#define DS_IRR_END_POLL_NS 1000
#endif
constexpr uint32_t kEndPollNs = DS_IRR_END_POLL_NS;
__device__ __forceinline__ bool mbar_wait_or_end(uint64_t* bar, uint32_t parity,
                                                 const volatile uint32_t* s_end, uint32_t k) {
    while (true) {
        if (mbar_try_wait(bar, parity, kEndPollNs)) return true;
        // Strictly beyond the end marker: the position holding the marker
        // itself still gets its arrival and must pass it on.
        if (*s_end < k) return false;
    }
}

template <class Op, bool PART>
__global__ void __launch_bounds__(kThreads, 1) irregular_kernel(const IrregParams p) {
    extern __shared__ __align__(128) uint32_t smem_raw[];
    // 128-byte aligned stage base (offset arithmetic keeps the shared window,
    // so the stage accesses stay LDS/STS)
    uint32_t* const smem = smem_raw + ((128u - (smem_addr(smem_raw) & 127u)) & 127u) / 4u;
    __shared__ __align__(8) uint64_t bar_full[kInStages], bar_free[kInStages];
    __shared__ __align__(8) uint64_t bar_drawn[kSlots], bar_counted[kSlots], bar_ranked[kSlots],
        bar_resolved[kSlots], bar_stored[kSlots];
    __shared__ SlotMeta meta[kSlots];
    __shared__ uint32_t s_epoch;
    __shared__ volatile uint32_t s_end;        // ring position of the end marker

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int s = 0; s < kInStages; ++s) {
            mbar_init(&bar_full[s], 1);
            mbar_init(&bar_free[s], 1);
        }
        for (int o = 0; o < kSlots; ++o) {
            mbar_init(&bar_drawn[o], 1);
            mbar_init(&bar_counted[o], 1);
            mbar_init(&bar_ranked[o], kGroupWarps);
            mbar_init(&bar_resolved[o], 1);
            mbar_init(&bar_stored[o], 1);
        }
        s_end = 0xffffffffu;
        mbar_fence_init();
    }
    __syncthreads();

    if (warp == kWarpProducer) {
        // ------------------------------------------------ producer (lane 0)
        if (lane != 0) return;
        uint32_t prev_t = kNoTile;
        for (uint32_t k = 0;; ++k) {
            const int s = k % kInStages, o = k % kSlots;
            uint32_t* stage = smem + s * kStageWords;
            mbar_wait(&bar_free[s], ((k / kInStages) & 1) ^ 1);  // rankers hold tile k - kInStages
            mbar_wait(&bar_stored[o], ((k / kSlots) & 1) ^ 1);   // slot o finished tile k - kSlots
            uint32_t t, epoch;
            draw_ticket(p.ctrl, p.draws, t, epoch);
            if (k == 0) s_epoch = epoch;
            if (t >= p.ntiles) {  // one failed draw per CTA ends its work
                meta[o].tile = kNoTile;
                s_end = k;
                mbar_arrive(&bar_drawn[o]);
                mbar_arrive(&bar_full[s]);
                return;
            }
            meta[o].tile = t;
            meta[o].prev_tile = prev_t;
            prev_t = t;
            mbar_arrive(&bar_drawn[o]);  // the resolver starts this tile's look-back now
            trace_event(p.trace, t, 0, globaltimer());
            trace_event(p.trace, t, 7, smid());
            debug_delay(t, 0);
            const uint64_t tb = uint64_t(t) * kT;
            uint64_t end = tb + kT < p.hi ? tb + kT : p.hi;
            end = (end + 3) & ~3ull;  // may read <= 12 bytes past the array end (same 16 B chunk)
            // Unique also needs the word before the tile: one copy starting 16
            // bytes early (measured faster than a separate 16-byte copy).
            const uint64_t beg = (Op::kUnique && t > 0) ? tb - kPre : tb;
            const uint32_t bytes = uint32_t(end - beg) * 4u;
            if (!DBG_NO_PFENCE) fence_proxy_async_smem();
            mbar_arrive_expect_tx(&bar_full[s], bytes);
            bulk_g2s(stage + kPre - (tb - beg), p.abase + beg, bytes, &bar_full[s]);
        }
    } else if (warp < kRankWarps) {
        // ------------------------------------------------ ranker warps
        // kRankGroups groups of kGroupWarps warps; group g ranks the tiles at
        // ring positions k = g (mod kRankGroups), so one group's barrier, scan
        // and status store overlap the other group's loads and ballots.
        const int g = warp / kGroupWarps, rw = warp % kGroupWarps;
        const int rt = tid - g * kRT;  // thread index within the group
        const uint32_t gbar = 1 + 2 * g;  // named barrier of the group (2 is the storers')
        const uint32_t lt = lanemask_lt();
        bool has_hprev = false;
        uint32_t hprev = 0;
        if (Op::kUnique) has_hprev = halo_prev(p, hprev);
        for (uint32_t k = g;; k += kRankGroups) {
            const int s = k % kInStages, o = k % kSlots;
            uint32_t* stage = smem + s * kStageWords;
            // the other group's end position releases this group too
            if (!mbar_wait_or_end(&bar_full[s], (k / kInStages) & 1, &s_end, k)) break;
            const uint32_t t = meta[o].tile;
            if (t == kNoTile) break;
            if (rt == 0) trace_event(p.trace, t, 1, globaltimer());
            if (DBG_SKIP_RANK) {  // timing experiment only
                named_bar_sync(gbar, kRT);
                if (rt == 0) {
                    meta[o].total = 0;
                    publish_status(status_ptr(p.status, t), make_status(t == 0 ? kStateIncl : kStateAgg, s_epoch, 0));
                    mbar_arrive(&bar_counted[o]);
                }
                if (lane == 0) mbar_arrive(&bar_ranked[o]);
                continue;
            }
            const uint64_t tb = uint64_t(t) * kT;
            const bool full = tb >= p.lo && tb + kT <= p.hi;

            // a3/a4: warp rw ranks tile words [xs, xs + kSeg) in kChunks chunks of
            // 32: lane l holds word x = xs + 32c + l of chunk c, so every shared
            // load and every compaction store below touches 32 consecutive words
            // (no bank conflicts), and a chunk's keep flags are one ballot.  The
            // ballot of chunk c is kept by lane c (one register instead of kChunks).
            const int xs = kSeg * rw;
            constexpr bool kMaskRegs = kChunks <= 16;  // else chunk c's mask is held by lane c
            constexpr bool kRc = kMaskRegs && !PART;  // chunk offsets from the count (registers)
            uint32_t v[kChunks];
            uint32_t mkr[kMaskRegs ? kChunks : 1], rc[kRc ? kChunks : 1];
            uint32_t mymask = 0;  // lane c: keep mask of chunk c (!kMaskRegs)
            uint32_t wrun = 0;    // kept words of the warp's segment
#pragma unroll
            for (int c = 0; c < kChunks; ++c) v[c] = stage[kPre + xs + 32 * c + lane];
            // Tile-relative bounds: only tile 0 (the array's first word, the lead
            // words below p.lo) and the last tile need the guarded pass; every
            // other tile takes the branch-free pass (same ops, no range checks).
            const uint32_t xlo = tb < p.lo ? uint32_t(p.lo - tb) : 0u;
            const uint32_t xhi = tb + kT <= p.hi ? uint32_t(kT) : uint32_t(p.hi - tb);
            const bool guarded = !full || t == 0;
            auto count_pass = [&](auto guard_tag) {
                constexpr bool G = decltype(guard_tag)::value;
#pragma unroll
                for (int c = 0; c < kChunks; ++c) {
                    const uint32_t x = uint32_t(xs + 32 * c + lane);
                    bool kp;
                    if constexpr (Op::kWide) {
                        // element = (even word, odd word) = lanes (2m, 2m+1) of the chunk
                        const uint32_t partner = __shfl_xor_sync(kFull, v[c], 1);
                        const uint32_t lo = (lane & 1) ? partner : v[c], hi = (lane & 1) ? v[c] : partner;
                        const uint32_t xe = x - (lane & 1);  // the element's first word
                        if constexpr (Op::kUnique) {
                            kp = lo != stage[kPre + xe - 2] || hi != stage[kPre + xe - 1];
                            if (G && t == 0 && xe == xlo) kp = true;  // the array's first element
                        } else {
                            kp = Op::keep2((uint64_t(hi) << 32) | lo, (uint64_t(p.value_hi) << 32) | p.value);
                        }
                    } else if constexpr (Op::kUnique) {
                        // previous word straight from the staged tile; x == 0 reads
                        // the word before the tile
                        kp = v[c] != stage[kPre + x - 1];
                        if (G && t == 0 && x == xlo) kp = !has_hprev || v[c] != hprev;  // the array's first word (R18)
                    } else {
                        kp = Op::keep(v[c], p.value);
                    }
                    if (G) kp = kp && x >= xlo && x < xhi;
                    const uint32_t mk = __ballot_sync(kFull, kp);
                    if constexpr (kMaskRegs) {
                        mkr[c] = mk;
                        if constexpr (kRc) rc[c] = wrun;  // kept words of the segment before chunk c
                    } else if (lane == c) {
                        mymask = mk;
                    }
                    wrun += __popc(mk);
                }
            };
            if (guarded) count_pass(std::true_type{});
            else count_pass(std::false_type{});
            if (lane == 0) meta[o].wtot[rw] = wrun;
            if (rt == 0) trace_event(p.trace, t, 13, globaltimer());
            named_bar_sync(gbar, kRT);  // warp totals written; every ranker holds its words
            if (DBG_EARLY_FREE && rt == 0) mbar_arrive(&bar_free[s]);  // timing experiment only
            if (rt == 0) trace_event(p.trace, t, 14, globaltimer());

            // Exclusive scan of the group's warp totals (input order), redundantly
            // in every warp.
            const uint32_t cw = lane < kGroupWarps ? meta[o].wtot[lane] : 0u;
            uint32_t iw = cw;
#pragma unroll
            for (int sh = 1; sh < kGroupWarps; sh <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, iw, sh);
                if (lane >= sh) iw += y;
            }
            const uint32_t total = __shfl_sync(kFull, iw, kGroupWarps - 1);
            const uint32_t wbase = __shfl_sync(kFull, iw - cw, rw);
            if (rt == 0) {
                // a4: publish the aggregate right away -- it depends on nothing else
                // (a relaxed status store).
                meta[o].total = total;
                debug_delay(t, 1);
                if (!DBG_NO_PUBLISH) publish_status(status_ptr(p.status, t), make_status(t == 0 ? kStateIncl : kStateAgg, s_epoch, total));
                trace_event(p.trace, t, 2, globaltimer());
                mbar_arrive(&bar_counted[o]);
            }

            // a6: compact the kept words in place, rank r -> stage[kPre + r]
            // (every ranker's words are in registers since the barrier).
            // Partition also places the false words, in input order, after the
            // trues: the f-th false word goes to stage[kPre + total + f], where
            // f = (valid words before it in the tile) - (true words before it).
            uint32_t* out = stage + kPre;
            const uint32_t vstart = tb < p.lo ? uint32_t(p.lo - tb) : 0u;  // invalid lead words (tile 0)
            uint32_t r = wbase;
#pragma unroll
            for (int c = 0; c < kChunks; ++c) {
                const uint32_t mk = kMaskRegs ? mkr[c] : __shfl_sync(kFull, mymask, c);
                if constexpr (kRc) r = wbase + rc[c];
                const uint32_t rl = r + __popc(mk & lt);  // trues before this word in the tile
                if constexpr (PART) {
                    // one (predicated) shared store per word: true -> rank, false -> after the trues
                    const uint32_t x = uint32_t(xs + 32 * c + lane);
                    const bool kb = mk >> lane & 1u;
                    const uint32_t idx = kb ? rl : total + (x - vstart) - rl;
                    const uint64_t e = tb + x;
                    if (kb || (!guarded || (e >= p.lo && e < p.hi))) out[idx] = v[c];
                } else if (mk >> lane & 1u) {
                    out[rl] = v[c];
                }
                if constexpr (!kRc) r += __popc(mk);
            }
            if (!DBG_NO_RFENCE) fence_proxy_async_smem();  // the compacted words leave through a bulk store
            __syncwarp();
            if (lane == 0) mbar_arrive(&bar_ranked[o]);  // this warp's part of the tile is compacted
            if (rt == 0) trace_event(p.trace, t, 15, globaltimer());
        }
    } else if (warp < kWarpStorer0) {
        // ------------------------------------------------ resolver warps
        const uint32_t r = warp - kWarpResolver0;
        for (uint32_t k = r;; k += kResolvers) {
            const int o = k % kSlots;
            const uint32_t use = k / kSlots;
            if (!mbar_wait_or_end(&bar_drawn[o], use & 1, &s_end, k)) break;
            const uint32_t t = meta[o].tile;
            if (t == kNoTile) {
                if (lane == 0) mbar_arrive(&bar_resolved[o]);
                break;
            }
            const uint32_t epoch = s_epoch;
            if (lane == 0) {
                debug_delay(t, 2);
                trace_event(p.trace, t, 3, globaltimer());
            }
            __syncwarp();
            // a5: the look-back needs only the ticket, so it runs while the tile is
            // still being loaded and ranked.
#ifdef DS_DEBUG_NO_LOOKBACK  // timing experiment only: wrong output, same traffic
            const uint64_t excl = uint64_t(t) * (kT / 2);
#else
            uint64_t excl = 0;
#if DS_IRR_LATE_LB  // experiment: start the look-back once the tile's own aggregate is out
            mbar_wait(&bar_counted[o], use & 1);
#endif
            if (t > 0) {
                const uint32_t tp = meta[o].prev_tile;
                if (kLocalChain && tp != kNoTile && t - tp - 1 <= uint32_t(32 * kLW))
                    excl = lookback_window(p.status, t, tp, &meta[(k + kSlots - 1) % kSlots], epoch, lane, p.trace);
                else
                    excl = lookback(p.status, t, epoch, lane, p.trace);
            }
#endif
            mbar_wait(&bar_counted[o], use & 1);  // the tile's aggregate is published
            const uint32_t total = meta[o].total;
            if (lane == 0) {
                meta[o].incl = excl + total;  // the CTA's next tile chains on this
                __threadfence_block();
                meta[o].incl_tile = t;
                if (t > 0 && !DBG_NO_PUBLISH) publish_status(status_ptr(p.status, t), make_status(kStateIncl, epoch, excl + total));
            }
            mbar_wait(&bar_ranked[o], use & 1);  // the compacted tile is in its stage
            if (lane == 0) {
                trace_event(p.trace, t, 4, globaltimer());
                meta[o].excl = excl;
                if (t == p.ntiles - 1 && p.d_out_n) *p.d_out_n = (excl + total) >> p.wshift;
                mbar_arrive(&bar_resolved[o]);
            }
        }
    } else {
        // ------------------------------------------------ storer warps
        // a7.  Kept words go out through one TMA bulk store per tile (the
        // aligned interior) plus <= 6 scalar head/tail words.  The stage is
        // first re-phased in shared memory so that its words sit at the same
        // 16-byte phase as their destination; the stage is released once the
        // bulk engine has read it.  Partition (two destinations) keeps the
        // register path (store_segment).
        const int st = tid - 32 * kWarpStorer0;
        for (uint32_t k = 0;; ++k) {
            const int o = k % kSlots;
            mbar_wait(&bar_resolved[o], (k / kSlots) & 1);
            const uint32_t t = meta[o].tile;
            if (t == kNoTile) break;
            if (st == 0) {
                trace_event(p.trace, t, 5, globaltimer());
                debug_delay(t, 3);
            }
            const int s_in = k % kInStages;
            uint32_t* const seg = smem + s_in * kStageWords + kPre;  // rank 0 (16-byte aligned)
            const uint32_t A = meta[o].total;
            const uint64_t tb0 = uint64_t(t) * kT;
            const uint64_t vs0 = tb0 > p.lo ? tb0 : p.lo;
            const uint64_t ve0 = tb0 + kT < p.hi ? tb0 + kT : p.hi;
            // Identity tile (in place, nothing removed in or before it): every
            // kept word would be written onto itself, so the stores are skipped.
            const bool identity = !PART && p.tbase == p.abase && meta[o].excl == vs0 - p.lo && A == ve0 - vs0;
#ifndef DS_DEBUG_NO_STORE  // timing experiment only: no output written
            // Bulk-store cnt words that sit at seg[off + r] (off % 4 == 0 or the
            // words before them are dead) to base[d0 + r]: re-phase them in shared
            // memory to d0's 16-byte phase, one TMA bulk store of the aligned
            // interior, scalar head and tail (<= 3 words each).
            auto bulk_segment = [&](uint32_t* base, uint64_t d0, uint32_t cnt, uint32_t off) {
                const uint64_t d1 = d0 + cnt;
                const uint32_t sh = (uint32_t(d0) - off) & 3u;  // shift that gives word r phase d0 + r
                uint32_t* const b = seg + (off & ~3u);          // aligned start of the moved block
                if (sh) rephase<kST>(b, cnt + (off & 3u), sh, st);  // word off + r -> off + sh + r
                const uint32_t* const w = seg + off + sh;        // word r now at w[r], phase of d0 + r
                const uint64_t g0 = (d0 + 3) & ~3ull, g1 = d1 & ~3ull;
                if (g1 > g0) {
                    fence_proxy_async_smem();  // re-phased words -> visible to the bulk engine
                    named_bar_sync(2, kST);
                    if (st == 0) bulk_s2g(base + g0, w + uint32_t(g0 - d0), uint32_t(g1 - g0) * 4u);
                    if (st < 3 && d0 + st < g0) stg_stream(base + d0 + st, w[st]);
                    if (st >= 3 && st < 6 && g1 + (st - 3) < d1)
                        stg_stream(base + g1 + (st - 3), w[uint32_t(g1 - d0) + (st - 3)]);
                } else {
                    named_bar_sync(2, kST);
                    if (uint32_t(st) < cnt) stg_stream(base + d0 + st, w[st]);  // cnt < 8
                }
            };
            if (!kBulkStore) {
                if (!identity) store_segment<kST>(p.tbase, p.tlo + meta[o].excl, A, seg, 0, st);
                if (PART) {
                    const uint64_t excl_f = (vs0 - p.lo) - meta[o].excl;
                    store_segment<kST>(p.fbase, p.flo + excl_f, uint32_t(ve0 - vs0) - A, seg, int32_t(A), st);
                }
            } else if (PART) {
                // Partition: trues at seg[0, A), falses at seg[A, A + F).  The trues'
                // re-phase writes whole 16-byte chunks, up to seg[A + 6), so the
                // first 7 falses are kept in registers until the trues' bulk store
                // has read the stage.
                const uint32_t F = uint32_t(ve0 - vs0) - A;
                const uint32_t keep7 = (uint32_t(st) < 7 && uint32_t(st) < F) ? seg[A + st] : 0u;
                named_bar_sync(2, kST);
                if (A > 0) bulk_segment(p.tbase, p.tlo + meta[o].excl, A, 0u);
                named_bar_sync(2, kST);
                if (st == 0) {
                    bulk_commit();
                    bulk_wait_read<0>();  // the trues have been read out of the stage
                }
                named_bar_sync(2, kST);
                if (uint32_t(st) < 7 && uint32_t(st) < F) seg[A + st] = keep7;
                named_bar_sync(2, kST);
                if (F > 0) bulk_segment(p.fbase, p.flo + ((vs0 - p.lo) - meta[o].excl), F, A);
            } else if (!identity && A > 0) {
                bulk_segment(p.tbase, p.tlo + meta[o].excl, A, 0u);
            }
#endif
            named_bar_sync(2, kST);  // every storer is done reading the stage
            if (st == 0) {
                trace_event(p.trace, t, 6, globaltimer());
                if (!DBG_NO_BULKWAIT) bulk_commit();        // (possibly empty) group of this tile
                if (!DBG_NO_BULKWAIT) bulk_wait_read<0>();  // the bulk engine has read the stage
                if (!DBG_EARLY_FREE) mbar_arrive(&bar_free[s_in]);
                mbar_arrive(&bar_stored[o]);
            }
        }
        if (st == 0) bulk_wait_all();  // the bulk stores are complete before the CTA exits
    }
}

struct LaunchCache {
    int dev = -1, sms = 0, per_sm = 0;
};

template <class Op, bool PART = false>
cudaError_t launch_op(IrregParams p, cudaStream_t s) {
    static thread_local LaunchCache lc;
    auto kern = irregular_kernel<Op, PART>;
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
    p.value_hi = a.value_hi;
    p.wshift = a.wide ? 1u : 0u;
    p.trace = debug_trace(p.ntiles);
    uint32_t* tptr = a.out_true ? a.out_true : a.ptr;
    const uint64_t tmis = (reinterpret_cast<uintptr_t>(tptr) >> 2) & 3u;
    p.tbase = tptr - tmis;
    p.tlo = tmis;
    if (a.out_false) {
        const uint64_t fmis = (reinterpret_cast<uintptr_t>(a.out_false) >> 2) & 3u;
        p.fbase = a.out_false - fmis;
        p.flo = fmis;
    }
    count_launch();
    const bool part = a.out_false != nullptr;
    if (a.wide) {
        switch (a.op) {
        case IrregOp::Compact: return launch_op<OpCompact64>(p, s);
        case IrregOp::Unique: return launch_op<OpUnique64>(p, s);
        case IrregOp::Select:
            switch (a.predicate) {
            case 0: return launch_op<OpSelect64<0>>(p, s);
            case 1: return launch_op<OpSelect64<1>>(p, s);
            case 2: return launch_op<OpSelect64<2>>(p, s);
            case 3: return launch_op<OpSelect64<3>>(p, s);
            case 4: return launch_op<OpSelect64<4>>(p, s);
            case 5: return launch_op<OpSelect64<5>>(p, s);
            case 6: return launch_op<OpSelect64<6>>(p, s);
            default: return cudaErrorInvalidValue;
            }
        }
        return cudaErrorInvalidValue;
    }
    switch (a.op) {
    case IrregOp::Compact: return launch_op<OpCompact>(p, s);
    case IrregOp::Unique: return launch_op<OpUnique>(p, s);
    case IrregOp::Select:
        switch (a.predicate) {
        case 0: return part ? launch_op<OpSelect<0>, true>(p, s) : launch_op<OpSelect<0>>(p, s);
        case 1: return part ? launch_op<OpSelect<1>, true>(p, s) : launch_op<OpSelect<1>>(p, s);
        case 2: return part ? launch_op<OpSelect<2>, true>(p, s) : launch_op<OpSelect<2>>(p, s);
        case 3: return part ? launch_op<OpSelect<3>, true>(p, s) : launch_op<OpSelect<3>>(p, s);
        case 4: return part ? launch_op<OpSelect<4>, true>(p, s) : launch_op<OpSelect<4>>(p, s);
        case 5: return part ? launch_op<OpSelect<5>, true>(p, s) : launch_op<OpSelect<5>>(p, s);
        case 6: return part ? launch_op<OpSelect<6>, true>(p, s) : launch_op<OpSelect<6>>(p, s);
        default: return cudaErrorInvalidValue;
        }
    }
    return cudaErrorInvalidValue;
}

}  // namespace ds
