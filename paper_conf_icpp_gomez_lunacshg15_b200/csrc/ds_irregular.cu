// ds_irregular.cu -- irregular Data Sliding on sm_100a: in-place, stable
// stream compaction, select and unique (Algorithm 2, P:168-190;
// §III-B; primitives §IV-B/C P:230-282).
//
// One persistent, warp-specialised CTA per SM walks input tiles of
// T = 8192 words in dynamic-ticket order (Fig. 4) through 4 input stages
// (partition: 6) and an output ring in shared memory.  Each role works on a different tile:
//
//   producer warp    a1 draws the next ticket as soon as an input stage and a
//                       slot are free; a2 loads the tile (plus, for unique,
//                       the words before it) with one TMA bulk copy (Alg. 2
//                       lines 1-11; "on-chip memory")
//  16 ranker warps   a3 keep flags (predicate / unique stencil), 4 bits
//                       per lane and 128-bit shared load; a4 the tile aggregate
//                       ("Reduction"), published as AGG at once; the
//                       input stage is released as soon as every ranker holds
//                       its words in registers; a6 rank of every kept word in
//                       input order ("binary prefix sum": one
//                       shuffle scan over packed per-lane counts) and the
//                       compaction of the kept words into the output ring
//   3 resolver warps a5 decoupled look-back over 32 predecessors per round
//                       trip, started as soon as the ticket is drawn, then
//                       INCL; the last tile writes out_n (a8).  This replaces
//                       the serial flag chain of Fig. 7, which is latency-bound
//                       on B200
//   2 x 2 storer     a7 re-phase the tile's ring region to the destination's
//     warps             16-byte phase, one TMA bulk store of [excl, excl + A)
//                       (scalar head/tail), then free the region once the bulk
//                       engine has read it; two groups on alternate tiles,
//                       regions released in ring order (partition: 2 x 3)
//
// A drawn tile's AGG depends only on its own load and ranking, never on the
// resolution of earlier tiles.  In-place safety: AGG/INCL
// are published only after the tile's words were read out of the copy; stores
// happen only after the look-back saw AGG/INCL of every lower tile; outputs
// of tile t lie in [0, (t+1)T), so no lower tile writes into a higher tile's
// input.  Deadlock freedom: look-backs wait only for lower (already drawn)
// tiles; a drawn tile reaches AGG without waiting on any other tile; a ranker
// waiting for ring space waits only for this CTA's lower tiles, whose
// aggregates (and so all their predecessors' statuses) are already out.
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
    uint64_t* trace_cta;  // diagnostics: per-CTA events (after the tiles' events), or null
    uint32_t* tbase;  // 16-byte-aligned base of the true/kept output (== abase in place)
    uint64_t tlo;     // its word offset (output word j lives at tbase[tlo + j])
    uint32_t* fbase;  // same for the false words (partition), or null
    uint64_t flo;
    uint64_t* const* pub_boards;  // peer count boards (sharded path), or null
    uint32_t pub_world, pub_rank;
    uint64_t pub_tag;
};

// a8 for a shard: the kept count goes straight into every rank's count board
// (peer memory over NVLink, mapped by CUDA IPC), one release store per rank,
// so no separate all-gather launch is needed (ds_shard_offsets_board reads it).
__device__ __forceinline__ void publish_to_boards(const IrregParams& p, uint64_t count) {
    const uint64_t w = board_word(count, p.pub_tag);
    for (uint32_t r = 0; r < p.pub_world; ++r) {
        uint64_t* slot = p.pub_boards[r] + 2 * p.pub_rank + (p.pub_tag & 1);
        asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(slot), "l"(w) : "memory");
    }
}

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

// ---- CTA shape ----------------------------------------------------------
// warps: 16 rankers (2 groups of 8) | 3 resolvers | 2 x 2 storers (2 x 3 for partition) | 1 producer
#ifndef DS_IRR_IN_STAGES
#define DS_IRR_IN_STAGES 4
#endif
#ifndef DS_IRR_SLOTS
#define DS_IRR_SLOTS 18
#endif
#ifndef DS_IRR_RESOLVERS
#define DS_IRR_RESOLVERS 3
#endif
#ifndef DS_IRR_STORE_WARPS
#define DS_IRR_STORE_WARPS 2
#endif
#ifndef DS_IRR_BULK_STORE
#define DS_IRR_BULK_STORE 1
#endif
constexpr bool kBulkStore = DS_IRR_BULK_STORE;  // a7 through TMA bulk stores (else 128-bit STG from registers)
#ifndef DS_IRR_RANK_GROUPS
#define DS_IRR_RANK_GROUPS 2
#endif
constexpr int kRankWarps = 16;
constexpr int kRankGroups = DS_IRR_RANK_GROUPS;   // ranker groups, each on its own tile
constexpr int kGroupWarps = kRankWarps / kRankGroups;
constexpr int kRT = 32 * kGroupWarps;     // threads of one ranker group
#ifndef DS_IRR_TILE
#define DS_IRR_TILE 8192
#endif
constexpr int kT = DS_IRR_TILE;           // words per tile (8192 = 32 KB)
constexpr int kSeg = kT / kGroupWarps;    // contiguous words ranked by one warp
constexpr int kRounds = kSeg / 128;       // rounds of 4 words per lane
constexpr int kPacks = (kRounds + 3) / 4; // registers of packed 8-bit round counts
static_assert(kRankGroups == 1 || kRankGroups == 2, "named barriers 1 and 3 serve the ranker groups");
// Every ranker lane arrives on the tile's "ranked" barrier after its own
// compaction stores (else lane 0 for the warp, after __syncwarp: the same
// ordering under the PTX model, but not one compute-sanitizer racecheck models).
#ifndef DS_IRR_ALL_LANES_ARRIVE
#define DS_IRR_ALL_LANES_ARRIVE 1
#endif
constexpr bool kAllLanesArrive = DS_IRR_ALL_LANES_ARRIVE;
constexpr int kRankedArrivals = kAllLanesArrive ? kRT : kGroupWarps;
static_assert(kRounds % 4 == 0, "whole packs of rounds");
constexpr int kInStages = DS_IRR_IN_STAGES;   // input tiles (TMA destination)
constexpr int kSlots = DS_IRR_SLOTS;          // tiles in flight per CTA (meta ring)
constexpr int kResolvers = DS_IRR_RESOLVERS;  // resolver r serves ring positions k = r mod kResolvers
#ifndef DS_IRR_PART_STORE_WARPS
#define DS_IRR_PART_STORE_WARPS 3
#endif
#ifndef DS_IRR_STORE_GROUPS
#define DS_IRR_STORE_GROUPS 2
#endif
#ifndef DS_IRR_PART_STORE_GROUPS
#define DS_IRR_PART_STORE_GROUPS 2
#endif
// Warp layout: rankers | resolvers | storers | producer.  The storers form
// kStoreGroups groups of kGroupStoreWarps warps; group g stores the tiles at
// ring positions k = g (mod kStoreGroups), so one group's per-tile fixed costs
// (re-phase, barriers, bulk issue, head / tail words) overlap the other's, and
// the regions are released in ring order (s_released).  Partition stores two
// segments per tile (trues and falses) and gets more storer warps.
template <bool PART>
struct Layout {
    static constexpr int kStoreGroups = PART ? DS_IRR_PART_STORE_GROUPS : DS_IRR_STORE_GROUPS;
    static constexpr int kGroupStoreWarps = PART ? DS_IRR_PART_STORE_WARPS : DS_IRR_STORE_WARPS;
    static constexpr int kStoreWarps = kStoreGroups * kGroupStoreWarps;
    static constexpr int kST = 32 * kGroupStoreWarps;  // threads of one storer group
    static_assert(kStoreGroups == 1 || kStoreGroups == 2, "named barriers 2 and 4 serve the storer groups");
    static constexpr int kWarpResolver0 = kRankWarps;
    static constexpr int kWarpStorer0 = kRankWarps + kResolvers;
    static constexpr int kWarpProducer = kWarpStorer0 + kStoreWarps;
    static constexpr int kThreads = 32 * (kWarpProducer + 1);
    static_assert(kThreads <= 1024, "CTA size");
#ifndef DS_IRR_REPHASE_CHUNKS
#define DS_IRR_REPHASE_CHUNKS 384
#endif
#ifndef DS_IRR_PART_REPHASE_CHUNKS
#define DS_IRR_PART_REPHASE_CHUNKS 384
#endif
    static constexpr int kRephaseChunks = PART ? DS_IRR_PART_REPHASE_CHUNKS : DS_IRR_REPHASE_CHUNKS;
    static constexpr int kRephaseU = kRephaseChunks / kST > 0 ? kRephaseChunks / kST : 1;
};
// Words before the tile in a stage (unique's boundary words).  Stages, and the
// tile inside each stage, start on 128-byte boundaries, so a bulk copy fills
// whole 128-byte shared-memory lines and unique's copy (which starts kPre
// words early) keeps a 128-byte aligned global source.
constexpr int kPre = 32;
constexpr int kStageWords = kT + kPre + 32;
// Output ring: the rankers compact each tile out of its input stage into the
// ring (the stage is free as soon as every ranker holds its words in
// registers); the storers drain the ring in tile order once the prefix is
// known.  Everything left of the 227 KB after the input stages.
constexpr int kStaticSmem = 128 * kSlots + 512;  // barriers + slot metadata (static shared memory; ptxas: 2304 B at 18 slots)
#ifndef DS_IRR_RING_WORDS
#define DS_IRR_RING_WORDS (((227 * 1024 - kStaticSmem - 128) / 4 - kInStages * kStageWords) / 32 * 32)
#endif
constexpr int kRingWords = DS_IRR_RING_WORDS;
constexpr size_t kSmem = (size_t(kInStages) * kStageWords + kRingWords) * 4 + 128;  // + alignment slack
// A ring region is one tile's kept words (+ its false words for partition),
// each rounded up to 4 words with 8 words of re-phase slack; a tile whose
// region does not fit (now) is compacted in place instead.
static_assert(kRingWords >= 0 && kRingWords % 4 == 0, "ring");
static_assert(kSlots >= kInStages, "a slot per input stage at least");
// Partition (true + false words: a region is a whole tile, which the ring
// rarely has room for, so its tiles stay in place) splits the same shared
// memory into more input stages and a smaller ring.
#ifndef DS_IRR_PART_STAGES
#define DS_IRR_PART_STAGES 6
#endif
template <bool PART>
struct SmemSplit {
    static constexpr int kFit = int((kSmem - 128) / 4) / kStageWords;  // stages the memory holds
    static constexpr int kStages = PART ? (DS_IRR_PART_STAGES < kFit ? DS_IRR_PART_STAGES : kFit) : kInStages;
    // the rest of the kernel's dynamic shared memory (the same size for both)
    static constexpr int kRingRaw = (int((kSmem - 128) / 4) - kStages * kStageWords) / 32 * 32;
    static constexpr int kRing = PART ? (kRingRaw > 0 ? kRingRaw : 0) : kRingWords;
    static_assert(kRing >= 0 && kStages * kStageWords + kRing <= int(kSmem / 4), "shared memory split");
    static_assert(kSlots >= kStages && kStages <= 32, "stages");
};
static_assert(kSlots % kResolvers == 0, "a slot is always served by the same resolver");
static_assert(kSlots % kRankGroups == 0 && kSlots % 2 == 0,
              "a slot is always served by the same ranker group and storer group");
static_assert(kSmem + kStaticSmem <= 227 * 1024, "shared memory");

struct SlotMeta {
    uint32_t tile;              // kNoTile: end of this CTA's work
    uint32_t stage;             // input stage holding the tile
    uint32_t total;             // kept words in the tile
    uint32_t freed_snap;        // ring words freed when the tile was counted
    unsigned long long excl;    // kept words in all lower tiles
    uint32_t ring_pos;          // ring word of the tile's rank 0 (multiple of 4), or kNoTile: in its stage
    uint32_t ring_end;          // ring allocation counter after this tile's decision (monotone)
    uint32_t ring_hpos;         // ring position after this tile's decision
    uint32_t wtot[kGroupWarps]; // kept words in each ranker warp's segment
};

__device__ __forceinline__ uint32_t round4(uint32_t x) { return (x + 3u) & ~3u; }
// ring words a tile occupies: kept words (+ false words, partition)
__device__ __forceinline__ uint32_t region_true(uint32_t total) { return total ? round4(total + 8u) : 0u; }
__device__ __forceinline__ uint32_t region_false(uint32_t falses) { return falses ? round4(falses + 8u) : 0u; }

__device__ __forceinline__ u32x4 lds_v4(uint32_t addr) {
    u32x4 r;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(addr));
    return r;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t addr) {
    uint32_t r;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(r) : "r"(addr));
    return r;
}
__device__ __forceinline__ void sts_u32(uint32_t addr, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
// Shared-memory flags between roles (the ring's free counter, the ring
// allocation order, the end marker), ordered at CTA scope: written with a
// release, read with an acquire.  Both are atomics (exchange / or 0) rather
// than st.release / ld.acquire: same ordering, and compute-sanitizer racecheck
// models atomics but not plain release/acquire accesses.
__device__ __forceinline__ void st_release_cta_smem(uint32_t* p, uint32_t v) {
    asm volatile("atom.release.cta.shared::cta.exch.b32 _, [%0], %1;" ::"r"(smem_addr(p)), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_cta_smem(const uint32_t* p) {
    uint32_t v;
    asm volatile("atom.acquire.cta.shared::cta.or.b32 %0, [%1], 0;" : "=r"(v) : "r"(smem_addr(p)) : "memory");
    return v;
}
// Free input stages (bit s): released (or) by the ranker / storer that is done
// reading the stage, claimed (and-not) by the producer only.
__device__ __forceinline__ void stage_release(uint32_t* mask, uint32_t s) {
    asm volatile("atom.release.cta.shared::cta.or.b32 _, [%0], %1;" ::"r"(smem_addr(mask)), "r"(1u << s)
                 : "memory");
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

// a5: decoupled look-back by one warp over 32 predecessors per round trip
// (one sector per status; a wider window reads more sectors per poll, a
// narrower one needs more round trips: DESIGN.md §7).  Lane l examines tile
// base - l.  Waits only for the tiles up to the nearest INCL predecessor; the
// nearest 32 AGG predecessors are re-read while polling (a nearer INCL ends
// the walk sooner).  Ends with one acquire fence per lane (strict build) and
// a __syncwarp so lane 0's later publication follows every lane's reads.
#ifndef DS_IRR_POLL_MIN
#define DS_IRR_POLL_MIN 64
#endif
#ifndef DS_IRR_POLL_MAX
#define DS_IRR_POLL_MAX 512
#endif
constexpr uint32_t kPollMinNs = DS_IRR_POLL_MIN;   // first back-off
constexpr uint32_t kPollMaxNs = DS_IRR_POLL_MAX;   // back-off cap
// Fault injection for the failure-detection test only: tile DS_DEBUG_DROP_TILE
// never publishes its status (as if its CTA were lost), so every later tile's
// look-back waits forever; built together with DS_SPIN_CAP_NS.
#ifndef DS_DEBUG_DROP_TILE
#define DS_DEBUG_DROP_TILE 0xffffffffu
#endif
constexpr uint32_t kDropTile = DS_DEBUG_DROP_TILE;
#ifndef DS_IRR_LATE_LB
#define DS_IRR_LATE_LB 0
#endif
constexpr int kLateLookback = DS_IRR_LATE_LB;  // look-back starts at: 0 the draw, 1 the own AGG, 2 the tile's landing
// L2 prefetch of the tile DS_IRR_PREFETCH grids ahead of each drawn ticket (0:
// off), while the CTA's last counted tile kept >= DS_IRR_PREFETCH_MIN_KEEP words
// (producer loop)
#ifndef DS_IRR_PREFETCH
#define DS_IRR_PREFETCH 1
#endif
constexpr uint32_t kPrefetchDist = DS_IRR_PREFETCH;
#ifndef DS_IRR_PART_PREFETCH
#define DS_IRR_PART_PREFETCH 0  // partition stores every word of a tile: no keep-fraction policy
#endif
#ifndef DS_IRR_PREFETCH_MIN_KEEP
#define DS_IRR_PREFETCH_MIN_KEEP 3686  // 45 % of a tile
#endif

__device__ __forceinline__ uint64_t lookback(uint64_t* __restrict__ status, uint32_t tile,
                                             uint32_t epoch, int lane, uint64_t* trace) {
    uint64_t excl = 0;
    uint32_t rounds = 0, polls = 0;
    int64_t base = int64_t(tile) - 1;
    uint32_t ns = kPollMinNs;
    SpinGuard guard;
    while (true) {
        int64_t idx = base - lane;
        uint64_t s = idx >= 0 ? ld_relaxed_gpu(status_ptr(status, idx)) : make_status(kStateIncl, epoch, 0);
        bool ok = status_current(s, epoch);
#ifndef DS_TRACE_PRODUCER
        if (rounds++ == 0 && lane == 0) trace_event(trace, tile, 10, globaltimer());
#else
        ++rounds;
#endif
        uint32_t L;  // nearest INCL at lane L (32: none this round)
        while (true) {
            const uint32_t inclm = __ballot_sync(kFull, ok && status_state(s) == kStateIncl);
            L = inclm ? uint32_t(__ffs(inclm) - 1) : 32u;
            const bool need = uint32_t(lane) <= L;  // every lane up to the nearest INCL
            if (!__any_sync(kFull, need && !ok)) break;
            guard.check("irregular look-back");
            __nanosleep(ns);
            ns = ns < kPollMaxNs ? ns * 2 : kPollMaxNs;
            ++polls;
            if (need && (!ok || status_state(s) != kStateIncl) && idx >= 0) {
                s = ld_relaxed_gpu(status_ptr(status, idx));
                ok = status_current(s, epoch);
            }
        }
        const uint32_t agg = uint32_t(lane) < L ? uint32_t(status_count(s)) : 0u;
        excl += uint64_t(__reduce_add_sync(kFull, agg));
        if (L < 32u) {
            excl += __shfl_sync(kFull, status_count(s), L);
            break;
        }
        base -= 32;
    }
#ifndef DS_TRACE_PRODUCER
    if (lane == 0) {
        trace_event(trace, tile, 8, rounds);
        trace_event(trace, tile, 9, polls);
        trace_event(trace, tile, 11, globaltimer());
    }
#endif
    lookback_acquire();
    __syncwarp();
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
// memory (ph = 1..3; seg 16-byte aligned with >= 6 writable words after the
// segment).  Destination chunk c (words
// [4c, 4c+4)) takes source words [4c-ph, 4c+4-ph): two aligned vector loads.
// Writing chunk c destroys sources of chunk c+1 only, so the chunks go in
// descending rounds, each reading everything before writing.
// kU chunks per thread per round: 384 chunks per round is the measured
// optimum for both 96 storers (kU = 4; compaction 1G f = 0.5: kU = 2 / 4 / 8
// 79.3 / 83.8 / 77.6 %) and 192 (partition, kU = 2: 75.7 %, kU = 4 73.6 %).
template <int kSTT, int kU>
__device__ __forceinline__ void rephase(uint32_t* seg, uint32_t cnt, uint32_t ph, int st, uint32_t bar) {
    const int32_t nchunks = int32_t((cnt + ph + 3) >> 2);
    for (int32_t hi = nchunks; hi > 0; hi -= kU * kSTT) {
        const int32_t lo = hi - kU * kSTT;
        u32x4 w[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int32_t c = lo + u * kSTT + st;
            if (c >= 0 && c < hi) {
                // chunk 0's leading words are dead (never stored): they are taken
                // from chunk 0 itself, since the words before seg may belong to
                // another tile's region
                const u32x4 a = *reinterpret_cast<const u32x4*>(seg + 4 * (c > 0 ? c : 1) - 4);
                const u32x4 b = *reinterpret_cast<const u32x4*>(seg + 4 * c);
                switch (ph) {  // uniform
                case 1: w[u] = u32x4{a.w, b.x, b.y, b.z}; break;
                case 2: w[u] = u32x4{a.z, a.w, b.x, b.y}; break;
                default: w[u] = u32x4{a.y, a.z, a.w, b.x}; break;
                }
            }
        }
        named_bar_sync(bar, kSTT);
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int32_t c = lo + u * kSTT + st;
            if (c >= 0 && c < hi) *reinterpret_cast<u32x4*>(seg + 4 * c) = w[u];
        }
        named_bar_sync(bar, kSTT);
    }
}

// a7 helper, one-barrier form of rephase(): every thread takes a contiguous
// run of m destination chunks (m odd, so the 16-byte accesses of 8
// neighbouring threads fall in distinct bank groups) and walks it downwards.
// Destination chunk c needs source chunks c-1 and c; writing it destroys
// source c only, which no lower chunk needs.  Within a run the walk order
// keeps every source intact until read; the one source a run needs from
// below its own range (chunk c_lo - 1, the next-lower run's top) is read
// before the barrier.  No barrier at the end: the caller's fence + barrier
// before the bulk store orders the writes.
#ifndef DS_IRR_STORE_WARP_SYNC
#define DS_IRR_STORE_WARP_SYNC 1
#endif
#ifndef DS_IRR_REPHASE_BATCH
#define DS_IRR_REPHASE_BATCH 4  // chunks read ahead per thread in rephase_runs (compaction, select, unique)
#endif
#ifndef DS_IRR_PART_REPHASE_BATCH
#define DS_IRR_PART_REPHASE_BATCH 2  // the same for partition (72 registers; measured 2 > 4 > 8)
#endif
#ifndef DS_IRR_REPHASE_RUNS
#define DS_IRR_REPHASE_RUNS 1
#endif
template <int kSTT, int kB>
__device__ __forceinline__ void rephase_runs(uint32_t* seg, uint32_t cnt, uint32_t ph, int st,
                                             uint32_t bar) {
    const int32_t nchunks = int32_t((cnt + ph + 3) >> 2);
    const int32_t m = ((nchunks + kSTT - 1) / kSTT) | 1;
    const int32_t c_lo = st * m;
    const int32_t c_hi = c_lo + m < nchunks ? c_lo + m : nchunks;
    // chunk 0's leading words are dead (never stored): its "lower" source is
    // chunk 0 itself, since the words before seg may belong to another region
    u32x4 below = u32x4{0u, 0u, 0u, 0u};
    if (c_lo < nchunks) below = *reinterpret_cast<const u32x4*>(seg + 4 * (c_lo > 0 ? c_lo - 1 : 0));
    named_bar_sync(bar, kSTT);
    if (c_lo >= c_hi) return;
    auto comb = [ph](const u32x4& a, const u32x4& b) {
        switch (ph) {  // uniform
        case 1: return u32x4{a.w, b.x, b.y, b.z};
        case 2: return u32x4{a.z, a.w, b.x, b.y};
        default: return u32x4{a.y, a.z, a.w, b.x};
        }
    };
    u32x4 cur = *reinterpret_cast<const u32x4*>(seg + 4 * (c_hi - 1));
    for (int32_t c = c_hi - 1; c >= c_lo; c -= kB) {
        u32x4 sv[kB];  // sources c-1 .. c-kB (all read before any of dests c .. c-kB+1 is written)
#pragma unroll
        for (int u = 0; u < kB; ++u) {
            const int32_t i = c - 1 - u;
            sv[u] = i >= c_lo ? *reinterpret_cast<const u32x4*>(seg + 4 * i) : below;
        }
#pragma unroll
        for (int u = 0; u < kB; ++u) {
            const int32_t d = c - u;
            if (d >= c_lo) *reinterpret_cast<u32x4*>(seg + 4 * d) = comb(sv[u], u ? sv[u - 1] : cur);
        }
        cur = sv[kB - 1];
    }
}

// mbarrier wait that also returns (false) once the CTA's work is known to
// end before ring position k (the resolvers take every kResolvers-th
// position, so the ones not holding the end marker are released this way).
// Suspend-time hint of those waits: it bounds how long a warp parked on a
// position past the end keeps the CTA (and so the launch) alive.
#ifndef DS_IRR_END_POLL_NS
#define DS_IRR_END_POLL_NS 1000
#endif
constexpr uint32_t kEndPollNs = DS_IRR_END_POLL_NS;
#ifndef DS_IRR_TESTWAIT
#define DS_IRR_TESTWAIT 1
#endif
__device__ __forceinline__ bool mbar_wait_or_end(uint64_t* bar, uint32_t parity,
                                                 const uint32_t* s_end, uint32_t k) {
    if (DS_IRR_TESTWAIT && mbar_test_wait(bar, parity)) return true;  // no suspension if already complete
    SpinGuard guard;
    while (true) {
        guard.check("irregular end-aware wait");
        if (mbar_try_wait(bar, parity, kEndPollNs)) return true;
        // Strictly beyond the end marker: the position holding the marker
        // itself still gets its arrival and must pass it on.
        if (ld_acquire_cta_smem(s_end) < k) return false;
    }
}

// a3: keep bits of the 4 words a lane holds in one round (bit j = word
// x0 + j), for 4-byte words.  pw = the word before x0 (unique).
template <class Op>
__device__ __forceinline__ uint32_t keep_bits4(const u32x4& v, uint32_t pw, uint32_t value) {
    if constexpr (Op::kUnique) {
        return uint32_t(v.x != pw) | uint32_t(v.y != v.x) << 1 | uint32_t(v.z != v.y) << 2 |
               uint32_t(v.w != v.z) << 3;
    } else {
        return uint32_t(Op::keep(v.x, value)) | uint32_t(Op::keep(v.y, value)) << 1 |
               uint32_t(Op::keep(v.z, value)) << 2 | uint32_t(Op::keep(v.w, value)) << 3;
    }
}
// Same for 8-byte elements (x, y) and (z, w): both words of an element get its
// flag.  (pz, pw) = the element before (x, y) (unique).
template <class Op>
__device__ __forceinline__ uint32_t keep_bits4_wide(const u32x4& v, uint32_t pz, uint32_t pw, uint64_t value) {
    bool k0, k1;
    if constexpr (Op::kUnique) {
        k0 = v.x != pz || v.y != pw;
        k1 = v.z != v.x || v.w != v.y;
    } else {
        k0 = Op::keep2(uint64_t(v.y) << 32 | v.x, value);
        k1 = Op::keep2(uint64_t(v.w) << 32 | v.z, value);
    }
    return (k0 ? 3u : 0u) | (k1 ? 12u : 0u);
}

template <class Op, bool PART>
__global__ void __launch_bounds__(Layout<PART>::kThreads, 1) irregular_kernel(const IrregParams p) {
    constexpr int kST = Layout<PART>::kST;
    constexpr int kWarpResolver0 = Layout<PART>::kWarpResolver0;
    constexpr int kWarpStorer0 = Layout<PART>::kWarpStorer0;
    constexpr int kWarpProducer = Layout<PART>::kWarpProducer;
    extern __shared__ __align__(128) uint32_t smem_raw[];
    // 128-byte aligned stage base (offset arithmetic keeps the shared window,
    // so the stage accesses stay LDS/STS)
    uint32_t* const smem = smem_raw + ((128u - (smem_addr(smem_raw) & 127u)) & 127u) / 4u;
    constexpr int kStagesK = SmemSplit<PART>::kStages;   // input stages of this kernel
    constexpr int kRingK = SmemSplit<PART>::kRing;       // output-ring words of this kernel
    uint32_t* const ring = smem + kStagesK * kStageWords;
    __shared__ __align__(8) uint64_t bar_loaded[kSlots], bar_drawn[kSlots], bar_counted[kSlots],
        bar_ranked[kSlots], bar_resolved[kSlots], bar_stored[kSlots];
    __shared__ SlotMeta meta[kSlots];
    __shared__ uint32_t s_epoch;
    __shared__ uint32_t s_end;           // ring position of the end marker (release / acquire)
    __shared__ uint32_t s_freed;         // output-ring words released by the storers (monotone)
    __shared__ uint32_t s_stages;        // free input stages (bit mask)
    __shared__ uint32_t s_alloc;         // ring positions whose ring decision is out
    __shared__ uint32_t s_released;      // ring positions whose regions are released (storer groups)
    __shared__ uint32_t s_recent_total;  // kept words of the CTA's most recently counted tile (prefetch policy)

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // per-CTA diagnostics: 0 entry, 1 initialised, 2 producer done, 3/4 storer
    // groups done, 5/6 ranker groups done, 7.. resolvers done; 15 SM id
    auto trace_cta = [&](int ev) { trace_event(p.trace_cta, blockIdx.x, ev, globaltimer()); };
    if (tid == 0) {
        trace_cta(0);
        trace_event(p.trace_cta, blockIdx.x, 15, smid());
    }
    // The producer warp sets up the barriers (one slot per lane) while its lane
    // 0's first ticket atomic (one L2 round trip) is in flight, then ARRIVES on
    // the start barrier and goes on to its first load; the other warps wait on
    // it (bar.arrive / bar.sync: the set-up is ordered before their accesses).
    unsigned long long first_old = 0;
    if (warp == kWarpProducer) {
        if (lane == 0) first_old = issue_ticket(p.ctrl);
        for (int o = lane; o < kSlots; o += 32) {
            mbar_init(&bar_loaded[o], 1);
            mbar_init(&bar_drawn[o], 1);
            mbar_init(&bar_counted[o], 1);
            mbar_init(&bar_ranked[o], kRankedArrivals);
            mbar_init(&bar_resolved[o], 1);
            mbar_init(&bar_stored[o], 1);
        }
        if (lane == 0) {
            s_end = 0xffffffffu;
            s_freed = 0;
            s_stages = (1u << kStagesK) - 1u;
            s_alloc = 0;
            s_released = 0;
            s_recent_total = 0;
        }
        if (lane < kSlots) mbar_fence_init();
        __syncwarp();
        named_bar_arrive(0, Layout<PART>::kThreads);
    } else {
        named_bar_sync(0, Layout<PART>::kThreads);
    }
    if (tid == 0) trace_cta(1);

    if (warp == kWarpProducer) {
        // ------------------------------------------------ producer (lane 0)
        if (lane != 0) return;
        // Free input stages: a tile compacted into the ring frees its stage at
        // once, one compacted in place only once stored.
        auto claim_stage = [&]() -> uint32_t {
            uint32_t m;
            SpinGuard guard;
            while ((m = ld_acquire_cta_smem(&s_stages)) == 0u) {
                guard.check("irregular producer stage wait");
                __nanosleep(32);
            }
            const uint32_t s = __ffs(m) - 1;
            atomicAnd(&s_stages, ~(1u << s));
            return s;
        };
        // Position k's ticket is drawn only once slot k and a stage are free, so a
        // drawn tile never waits for anything but its own load (a drawn tile that
        // waited would hold up every later tile's look-back: a convoy; drawing
        // the next ticket as soon as a second stage is free measured -3 to -7 %,
        // DESIGN.md §7).
        uint64_t claim_cur = p.trace ? globaltimer() : 0;  // diagnostics: stage wait start
        uint32_t s_cur = claim_stage();
        unsigned long long old_cur = first_old;  // issued at kernel entry
        bool pf_on = DS_IRR_PREFETCH_MIN_KEEP == 0;  // L2 prefetch policy (see the end of the loop)
        for (uint32_t k = 0;; ++k) {
            const int o = k % kSlots;
            const uint32_t s = s_cur;
            const uint64_t t_claim = claim_cur;
            uint32_t* stage = smem + s * kStageWords;
            uint32_t t, epoch;
            take_ticket(p.ctrl, p.draws, old_cur, t, epoch);
#ifdef DS_TRACE_PRODUCER
            const uint64_t tp_taken = globaltimer();
#endif
            if (k == 0) s_epoch = epoch;
            if (t >= p.ntiles) {  // a failed draw ends the CTA's work
                meta[o].tile = kNoTile;
                st_release_cta_smem(&s_end, k);
                mbar_arrive(&bar_drawn[o]);
                mbar_arrive(&bar_loaded[o]);
                // End markers for the other resolvers' (and ranker groups') next
                // positions, so each of them finds one and no warp has to poll
                // for the end of the work.
                static_assert(kRankGroups <= kResolvers, "end markers");
                for (uint32_t j = 1; j < uint32_t(kResolvers); ++j) {
                    const uint32_t kj = k + j, oj = kj % kSlots;
                    mbar_wait(&bar_stored[oj], ((kj / kSlots) & 1) ^ 1);
                    meta[oj].tile = kNoTile;
                    mbar_arrive(&bar_drawn[oj]);
                    if (j < uint32_t(kRankGroups)) mbar_arrive(&bar_loaded[oj]);
                }
                trace_cta(2);
                return;
            }
            meta[o].tile = t;
            meta[o].stage = s;
            mbar_arrive(&bar_drawn[o]);  // the resolver starts this tile's look-back now
            trace_event(p.trace, t, 0, globaltimer());
            trace_event(p.trace, t, 7, smid());
            trace_event(p.trace, t, 13, t_claim);  // start of the wait for a free input stage
            debug_delay(t, 0);
            const uint64_t tb = uint64_t(t) * kT;
            const uint64_t end = tb + kT < p.hi ? tb + kT : p.hi;
            // The bulk copy covers whole 16-byte chunks from the tile's aligned
            // start: tile 0 also reads the (lo) words before ptr, which share
            // ptr's 16-byte chunk.  It stops at the last whole chunk of the
            // array; the 1..3 words after it (last tile only) are loaded by this
            // thread, so nothing past the array's end is read (include/ds.h).
            const uint64_t end16 = end & ~3ull;
            // Unique also needs the word before the tile: one copy starting kPre
            // words early (measured faster than a separate 16-byte copy).
            const uint64_t beg = (Op::kUnique && t > 0) ? tb - kPre : tb;
            uint32_t* const dst = stage + kPre - (tb - beg);
            for (uint64_t w = end16 > beg ? end16 : beg; w < end; ++w)
                dst[w - beg] = ldg_stream(p.abase + w);  // before the arrival that publishes the stage
            const uint32_t bytes = end16 > beg ? uint32_t(end16 - beg) * 4u : 0u;
#ifdef DS_TRACE_PRODUCER  // producer sub-steps in slots 8-11 (the look-back's diagnostics are off)
            trace_event(p.trace, t, 8, tp_taken);
            trace_event(p.trace, t, 9, globaltimer());
#endif
            fence_proxy_async_smem();
#ifdef DS_TRACE_PRODUCER
            trace_event(p.trace, t, 10, globaltimer());
#endif
            mbar_arrive_expect_tx(&bar_loaded[o], bytes);
            if (bytes) bulk_g2s(dst, p.abase + beg, bytes, &bar_loaded[o]);
#ifdef DS_TRACE_PRODUCER
            trace_event(p.trace, t, 11, globaltimer());
#endif
            if (kPrefetchDist && (PART ? DS_IRR_PART_PREFETCH : pf_on)) {
                // L2 prefetch of the tile kPrefetchDist grids ahead: tickets are drawn
                // in order by all CTAs, so that tile is drawn ~1-3 us from now and its
                // load then hits L2 (each tile is prefetched once, by the CTA that drew
                // the ticket kPrefetchDist * grid before it).  No lower tile ever
                // writes into a higher tile's input (§4.3), so the lines stay current.
                const uint64_t tp = uint64_t(t) + uint64_t(kPrefetchDist) * gridDim.x;
                if (tp < p.ntiles) {
                    const uint64_t pb = tp * kT - ((Op::kUnique && tp > 0) ? kPre : 0);
                    const uint64_t pe = (tp * kT + kT < p.hi ? tp * kT + kT : p.hi) & ~3ull;
                    if (pe > pb) bulk_prefetch_l2(p.abase + pb, uint32_t(pe - pb) * 4u);
                }
            }
            // the next position's ticket: once its slot and a stage are free
            {
                const uint32_t k1 = k + 1, o1 = k1 % kSlots;
                mbar_wait(&bar_stored[o1], ((k1 / kSlots) & 1) ^ 1);  // slot o1 finished tile k1 - kSlots
                claim_cur = p.trace ? globaltimer() : 0;
                s_cur = claim_stage();
                old_cur = issue_ticket(p.ctrl);
            }
            // The prefetch policy for the next tile, decided off the critical path
            // (the next ticket's round trip is in flight): prefetch only while the
            // CTA's last counted tile kept >= DS_IRR_PREFETCH_MIN_KEEP words.  At
            // low keep fractions the producer loop, not the input stages, bounds
            // the rate, and the prefetch does not pay.
            if (kPrefetchDist && DS_IRR_PREFETCH_MIN_KEEP)
                pf_on = *static_cast<volatile uint32_t*>(&s_recent_total) >= uint32_t(DS_IRR_PREFETCH_MIN_KEEP);
        }
    } else if (warp < kRankWarps) {
        // ------------------------------------------------ ranker warps
        // kRankGroups groups of kGroupWarps warps; group g ranks the tiles at ring
        // positions k = g (mod kRankGroups), so one group's shuffle-scan chains and
        // barrier overlap the other group's loads and stores.  Warp rw of a group
        // ranks tile words [xs, xs + kSeg) in rounds of 128: in round r lane l
        // holds the 4 words xs + 128r + 4l + {0..3} (one 128-bit shared load,
        // conflict-free).  Keep flags are 4 bits per lane and round (a3), counted
        // per lane; 4 rounds' counts travel in 8-bit fields of one register
        // through ONE shuffle scan over the lanes, which gives every lane its
        // exclusive offset in those rounds at once (a4/a6).  No ballot and no
        // per-word POPC: those run at a quarter of the ALU rate and bound the
        // chunked ballot ranker.
        const int g = warp / kGroupWarps, rw = warp % kGroupWarps;
        const int rt = tid - g * kRT;         // thread index within the group
        // named barrier of the group (2 and 4 are the storers').  A register
        // id here: one copy of the ranker loop per group (immediate ids) doubles
        // the ranker code and measured -9 % at f = 0.5.
        const uint32_t gbar = 1 + 2 * g;
        const int xs = kSeg * rw;
        const uint32_t smem_b = smem_addr(smem);
        const uint32_t ring_b = smem_addr(ring);
        bool has_hprev = false;
        uint32_t hprev = 0;
        if (Op::kUnique && !Op::kWide) has_hprev = halo_prev(p, hprev);
        for (uint32_t k = g;; k += kRankGroups) {
            const int o = k % kSlots;
            if (!mbar_wait_or_end(&bar_loaded[o], (k / kSlots) & 1, &s_end, k)) {
                if (rt == 0) trace_cta(5 + g);
                break;
            }
            const uint32_t t = meta[o].tile;
            if (t == kNoTile) {
                if (rt == 0) trace_cta(5 + g);
                break;
            }
            const uint32_t s = meta[o].stage;
            if (rt == 0) trace_event(p.trace, t, 1, globaltimer());
            const uint64_t tb = uint64_t(t) * kT;
            const bool full = tb >= p.lo && tb + kT <= p.hi;
            // Tile-relative valid range: only tile 0 (lead words below p.lo) and the
            // last tile need range checks.
            const uint32_t xlo = tb < p.lo ? uint32_t(p.lo - tb) : 0u;
            const uint32_t xhi = tb + kT <= p.hi ? uint32_t(kT) : uint32_t(p.hi - tb);
            const bool guarded = !full || t == 0;
            const uint32_t st_b = smem_b + 4u * (s * uint32_t(kStageWords) + kPre);  // tile word 0
            u32x4 v[kRounds];
#pragma unroll
            for (int r = 0; r < kRounds; ++r) v[r] = lds_v4(st_b + 4u * uint32_t(xs + 128 * r + 4 * lane));
            uint32_t kb = 0, P[kPacks];
#pragma unroll
            for (int i = 0; i < kPacks; ++i) P[i] = 0;
            // Keep bits of all rounds.  Only tile 0 (the array's first word, lead
            // words before ptr) and the last tile need range checks: the guarded
            // variant is a separate, compile-time copy, so every other tile runs
            // the pass without a per-round branch.
            auto keep_pass = [&](auto guard_tag) {
                constexpr bool G = decltype(guard_tag)::value;
                // unique: lane l-1's last word of round r; lane 0 receives lane 31's,
                // which is lane 0's predecessor in round r+1 (one shuffle per round)
                uint32_t rot_z = 0, rot_w = 0;
#pragma unroll
                for (int r = 0; r < kRounds; ++r) {
                    const uint32_t x0 = uint32_t(xs + 128 * r + 4 * lane);
                    uint32_t b;
                    if constexpr (Op::kWide) {
                        uint32_t pz = 0, pw = 0;
                        if constexpr (Op::kUnique) {
                            // element before (x, y): lane l-1's (z, w), lane 31 of the previous
                            // round, or the two staged words before the segment
                            const uint32_t tz = __shfl_sync(kFull, v[r].z, (lane + 31) & 31);
                            const uint32_t tw = __shfl_sync(kFull, v[r].w, (lane + 31) & 31);
                            if (lane != 0) {
                                pz = tz, pw = tw;
                            } else if (r > 0) {
                                pz = rot_z, pw = rot_w;
                            } else {
                                pz = lds_u32(st_b + 4u * uint32_t(xs - 2));
                                pw = lds_u32(st_b + 4u * uint32_t(xs - 1));
                            }
                            rot_z = tz, rot_w = tw;
                        }
                        b = keep_bits4_wide<Op>(v[r], pz, pw, uint64_t(p.value_hi) << 32 | p.value);
                        if (Op::kUnique && G && t == 0) {  // the array's first element is kept
                            if (x0 == xlo) b |= 3u;
                            if (x0 + 2 == xlo) b |= 12u;
                        }
                    } else {
                        uint32_t pw = 0;
                        if constexpr (Op::kUnique) {
                            // word before x0: lane l-1's last word, lane 31 of the previous
                            // round, or the staged word before the segment (P:280 for xs = 0)
                            const uint32_t tw = __shfl_sync(kFull, v[r].w, (lane + 31) & 31);
                            pw = lane != 0 ? tw : r > 0 ? rot_w : lds_u32(st_b + 4u * uint32_t(xs - 1));
                            rot_w = tw;
                        }
                        b = keep_bits4<Op>(v[r], pw, p.value);
                        if (Op::kUnique && G && t == 0 && x0 <= xlo && xlo < x0 + 4) {
                            // the array's first word (R18): kept unless it equals the halo word
                            const uint32_t j = xlo - x0;
                            const uint32_t w0 = j == 0 ? v[r].x : j == 1 ? v[r].y : j == 2 ? v[r].z : v[r].w;
                            const bool k0 = !has_hprev || w0 != hprev;
                            b = (b & ~(1u << j)) | (uint32_t(k0) << j);
                        }
                    }
                    if (G) {
                        // words outside [xlo, xhi) are not elements of the array
                        const uint32_t lo_ok = x0 >= xlo ? 15u : (15u << (xlo - x0)) & 15u;
                        const uint32_t hi_ok = x0 + 4 <= xhi ? 15u : x0 >= xhi ? 0u : (1u << (xhi - x0)) - 1u;
                        b &= lo_ok & hi_ok;
                    }
                    kb |= b << (4 * r);
                    P[r / 4] += uint32_t(__popc(b)) << (8 * (r % 4));
                }
            };
            if (guarded) keep_pass(std::true_type{});
            else keep_pass(std::false_type{});
            // exclusive offsets of every lane in all rounds (8-bit fields, <= 128 each)
            uint32_t inc[kPacks];
#pragma unroll
            for (int i = 0; i < kPacks; ++i) inc[i] = P[i];
#pragma unroll
            for (int sh = 1; sh < 32; sh <<= 1) {
#pragma unroll
                for (int i = 0; i < kPacks; ++i) {
                    const uint32_t y = __shfl_up_sync(kFull, inc[i], sh);
                    if (lane >= sh) inc[i] += y;
                }
            }
            uint32_t E[kPacks], R[kRounds];  // R[r]: kept words of the segment before round r
            uint32_t wrun = 0;               // kept words of the warp's segment
#pragma unroll
            for (int i = 0; i < kPacks; ++i) {
                E[i] = inc[i] - P[i];
                const uint32_t T4 = __shfl_sync(kFull, inc[i], 31);
#pragma unroll
                for (int f = 0; f < 4; ++f) {
                    R[4 * i + f] = wrun;
                    wrun += T4 >> (8 * f) & 255u;
                }
            }
            if (lane == 0) meta[o].wtot[rw] = wrun;
            if (rt == 0) {
                meta[o].freed_snap = ld_acquire_cta_smem(&s_freed);  // one ring view for the group
            }
            named_bar_sync(gbar, kRT);  // warp totals written; every ranker holds its words
            if (rt == 0) trace_event(p.trace, t, 14, globaltimer());
            // Exclusive scan of the warp totals (input order), redundantly in every warp.
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
                if (kPrefetchDist && DS_IRR_PREFETCH_MIN_KEEP)
                    *static_cast<volatile uint32_t*>(&s_recent_total) = total;  // a hint only
                debug_delay(t, 1);
                if (t != kDropTile)
                    publish_status(status_ptr(p.status, t), make_status(t == 0 ? kStateIncl : kStateAgg, s_epoch, total));
                trace_event(p.trace, t, 2, globaltimer());
                mbar_arrive(&bar_counted[o]);
            }
            // Where the compacted tile waits for its prefix: a region of the output
            // ring if the ring has room (the input stage is then free at once), else
            // in place in its input stage (held until stored).  Rankers never wait
            // for ring space: a blocked ranker would keep drawn tiles from
            // publishing their aggregates and stall every look-back behind them.
            // Ring regions are allocated in ring-position order: position k starts
            // from position k-1's allocation state (meta of the previous slot, valid
            // once s_alloc reaches k); every thread of the group computes the same
            // decision from the same snapshot.
            uint32_t h = 0, hp = 0;
            if (k > 0) {
                if (kRankGroups > 1) {
                    if (lane == 0)
                        for (SpinGuard guard; ld_acquire_cta_smem(&s_alloc) < k;) {
                            guard.check("irregular ring allocation order");
                            __nanosleep(32);
                        }
                    __syncwarp();
                }
                const SlotMeta& pm = meta[(k + kSlots - 1) % kSlots];
                h = pm.ring_end;
                hp = pm.ring_hpos;
            }
            const uint32_t falses = PART ? (xhi - xlo) - total : 0u;
            const uint32_t need_t = region_true(total);
            const uint32_t need = need_t + region_false(falses);
            const uint32_t h0 = h, hp0 = hp;
            if (hp + need > uint32_t(kRingK)) {  // no wrapped regions: skip the ring's end
                h += uint32_t(kRingK) - hp;
                hp = 0;
            }
            const bool in_ring = h + need - meta[o].freed_snap <= uint32_t(kRingK);
            const uint32_t rpos = hp;
            if (rt == 0) {
                meta[o].ring_pos = in_ring ? rpos : kNoTile;
                trace_event(p.trace, t, 7, smid() | uint64_t(in_ring) << 16);  // diagnostics: ring or in place
                meta[o].ring_end = in_ring ? h + need : h0;
                meta[o].ring_hpos = in_ring ? hp + need : hp0;
                if (kRankGroups > 1) st_release_cta_smem(&s_alloc, k + 1);
                if (in_ring) stage_release(&s_stages, s);  // every ranker of the group holds its words
            }
            // a6: compact the kept words, rank r -> out[r] (partition: the f-th false
            // word -> out[need_t + f]), out = ring + rpos or the tile's stage.
            if (PART || wrun != 0) {
                const uint32_t out_b = in_ring ? ring_b + 4u * rpos : st_b;
#pragma unroll
                for (int r = 0; r < kRounds; ++r) {
                    const uint32_t b = kb >> (4 * r) & 15u;
                    const uint32_t q0 = wbase + R[r] + (E[r / 4] >> (8 * (r % 4)) & 255u);  // trues before word x0
                    const uint32_t q1 = q0 + (b & 1u), q2 = q1 + (b >> 1 & 1u), q3 = q2 + (b >> 2 & 1u);
                    if constexpr (PART) {
                        // one (predicated) shared store per valid word: true -> its rank,
                        // false -> after the trues' region, in input order
                        const uint32_t x0 = uint32_t(xs + 128 * r + 4 * lane);
                        const uint32_t fb = need_t + x0 - xlo;  // + (valid words before x0) - trues before
                        const uint32_t q[4] = {q0, q1, q2, q3};
                        const uint32_t w[4] = {v[r].x, v[r].y, v[r].z, v[r].w};
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            const uint32_t x = x0 + j;
                            const bool kt = b >> j & 1u;
                            const uint32_t idx = kt ? q[j] : fb + j - q[j];
                            if (kt || !guarded || (x >= xlo && x < xhi)) sts_u32(out_b + 4u * idx, w[j]);
                        }
                    } else {
                        if (b & 1u) sts_u32(out_b + 4u * q0, v[r].x);
                        if (b & 2u) sts_u32(out_b + 4u * q1, v[r].y);
                        if (b & 4u) sts_u32(out_b + 4u * q2, v[r].z);
                        if (b & 8u) sts_u32(out_b + 4u * q3, v[r].w);
                    }
                }
                fence_proxy_async_smem();  // the compacted words leave through a bulk store
            }
            if (kAllLanesArrive) {
                mbar_arrive(&bar_ranked[o]);  // each lane's compaction stores are released by its own arrival
            } else {
                __syncwarp();
                if (lane == 0) mbar_arrive(&bar_ranked[o]);  // this warp's part of the tile is compacted
            }
            if (rt == 0) trace_event(p.trace, t, 15, globaltimer());
        }
    } else if (warp < kWarpStorer0) {
        // ------------------------------------------------ resolver warps
        const uint32_t r = warp - kWarpResolver0;
        for (uint32_t k = r;; k += kResolvers) {
            const int o = k % kSlots;
            const uint32_t use = k / kSlots;
            mbar_wait(&bar_drawn[o], use & 1);  // a tile, or an end marker (every resolver gets one)
            const uint32_t t = meta[o].tile;
            if (t == kNoTile) {
                if (lane == 0) {
                    mbar_arrive(&bar_resolved[o]);
                    trace_cta(7 + r);
                }
                break;
            }
            const uint32_t epoch = s_epoch;
            if (lane == 0) {
                debug_delay(t, 2);
                trace_event(p.trace, t, 3, globaltimer());
            }
            __syncwarp();
            // a5: the look-back needs only the ticket, so it starts at once (with
            // two storer groups this beats starting at the own AGG, DS_IRR_LATE_LB=1,
            // by 2 % at f = 0.5 and 3 % at f = 0.9; -1.3 % at f = 0).
            if (kLateLookback == 1) mbar_wait(&bar_counted[o], use & 1);
            if (kLateLookback == 2) mbar_wait(&bar_loaded[o], use & 1);
            // (64 / 128 statuses per round trip instead of 32 measured -1 to -6 %)
            const uint64_t excl = t > 0 ? lookback(p.status, t, epoch, lane, p.trace) : 0ull;
            if (kLateLookback != 1) mbar_wait(&bar_counted[o], use & 1);  // the tile's aggregate is published
            const uint32_t total = meta[o].total;
            if (lane == 0 && t > 0 && t != kDropTile)
                publish_status(status_ptr(p.status, t), make_status(kStateIncl, epoch, excl + total));
            mbar_wait(&bar_ranked[o], use & 1);  // the compacted tile is in the ring
            if (lane == 0) {
                trace_event(p.trace, t, 4, globaltimer());
                meta[o].excl = excl;
                if (t == p.ntiles - 1) {  // a8
                    if (p.d_out_n) *p.d_out_n = (excl + total) >> p.wshift;
                    if (p.pub_boards) publish_to_boards(p, (excl + total) >> p.wshift);
                }
                mbar_arrive(&bar_resolved[o]);
            }
        }
    } else {
        // ------------------------------------------------ storer warps
        // a7.  A tile's ring region goes out through one TMA bulk store (the
        // aligned interior) plus <= 6 scalar head/tail words: the region is first
        // re-phased in shared memory so its words sit at their destination's
        // 16-byte phase.  The region is released once the bulk engine has read it.
        constexpr int kSG = Layout<PART>::kStoreGroups;
        const int sg = (tid - 32 * kWarpStorer0) / kST;  // storer group
        const int st = (tid - 32 * kWarpStorer0) % kST;  // thread within the group
        // one compiled copy of the loop per group, so the group's named barrier
        // id is an immediate (a register id measured -12 % at f = 0.5)
        auto storer_loop = [&](auto sg_tag) {
        constexpr uint32_t kG = decltype(sg_tag)::value;
        constexpr uint32_t sbar = kG ? 4u : 2u;         // the group's named barrier
        for (uint32_t k = kG;; k += kSG) {
            const int o = k % kSlots;
            mbar_wait(&bar_resolved[o], (k / kSlots) & 1);
            const uint32_t t = meta[o].tile;
            if (t == kNoTile) break;
            if (st == 0) {
                trace_event(p.trace, t, 5, globaltimer());
                debug_delay(t, 3);
            }
            const uint32_t A = meta[o].total;
            const uint64_t excl = meta[o].excl;
            const uint32_t rpos = meta[o].ring_pos;
            const bool in_ring = rpos != kNoTile;
            uint32_t* const seg = in_ring ? ring + rpos : smem + meta[o].stage * kStageWords + kPre;
            const uint32_t ring_end = meta[o].ring_end;
            const uint64_t tb0 = uint64_t(t) * kT;
            const uint64_t vs0 = tb0 > p.lo ? tb0 : p.lo;
            const uint64_t ve0 = tb0 + kT < p.hi ? tb0 + kT : p.hi;
            // Identity tile (in place, nothing removed in or before it): every kept
            // word would be written onto itself, so the stores are skipped.
            const bool identity = !PART && p.tbase == p.abase && p.tlo == p.lo && excl == vs0 - p.lo &&
                                  A == ve0 - vs0;
            // Bulk-store the cnt words w0[0, cnt) (16-byte aligned) to base[d0, d0 + cnt).
            auto bulk_segment = [&](uint32_t* w0, uint32_t* base, uint64_t d0, uint32_t cnt) {
                const uint64_t d1 = d0 + cnt;
                const uint32_t sh = uint32_t(d0) & 3u;  // word r must sit at phase (d0 + r) & 3
                if (sh) {
                    if (DS_IRR_REPHASE_RUNS) rephase_runs<kST, PART ? DS_IRR_PART_REPHASE_BATCH : DS_IRR_REPHASE_BATCH>(w0, cnt, sh, st, sbar);
                    else rephase<kST, Layout<PART>::kRephaseU>(w0, cnt, sh, st, sbar);
                }
                const uint32_t* const w = w0 + sh;
                const uint64_t g0 = (d0 + 3) & ~3ull, g1 = d1 & ~3ull;
#ifdef DS_TRACE_STORER
                if (st == 0) trace_event(p.trace, t, 8, globaltimer());
#endif
                if (g1 > g0) {
                    fence_proxy_async_smem();  // re-phased words -> visible to the bulk engine
#ifdef DS_TRACE_STORER
                    if (st == 0) trace_event(p.trace, t, 9, globaltimer());
#endif
                    named_bar_sync(sbar, kST);
#ifdef DS_TRACE_STORER
                    if (st == 0) trace_event(p.trace, t, 10, globaltimer());
#endif
                    if (st == 0) bulk_s2g(base + g0, w + uint32_t(g0 - d0), uint32_t(g1 - g0) * 4u);
#ifdef DS_TRACE_STORER
                    if (st == 0) trace_event(p.trace, t, 11, globaltimer());
#endif
                    if (st < 3 && d0 + st < g0) stg_stream(base + d0 + st, w[st]);
                    if (st >= 3 && st < 6 && g1 + (st - 3) < d1)
                        stg_stream(base + g1 + (st - 3), w[uint32_t(g1 - d0) + (st - 3)]);
                } else {
                    named_bar_sync(sbar, kST);
                    if (uint32_t(st) < cnt) stg_stream(base + d0 + st, w[st]);  // cnt < 8
                }
            };
            if (!kBulkStore) {
                if (!identity) store_segment<kST>(p.tbase, p.tlo + excl, A, seg, 0, st);
                if constexpr (PART)
                    store_segment<kST>(p.fbase, p.flo + ((vs0 - p.lo) - excl), uint32_t(ve0 - vs0) - A, seg,
                                       int32_t(region_true(A)), st);
            } else {
                if (!identity && A > 0) bulk_segment(seg, p.tbase, p.tlo + excl, A);
                if constexpr (PART) {
                    const uint32_t F = uint32_t(ve0 - vs0) - A;
                    if (F > 0) bulk_segment(seg + region_true(A), p.fbase, p.flo + ((vs0 - p.lo) - excl), F);
                }
            }
            // Every storer is done with the region.  With bulk stores only warp 0's
            // lanes 0..7 (the scalar head / tail words) read it after the last
            // barrier, so a warp sync orders them before lane 0's release.
            if (kBulkStore && DS_IRR_STORE_WARP_SYNC) {
                if (st < 32) __syncwarp();
            } else {
                named_bar_sync(sbar, kST);
            }
            if (st == 0) {
                trace_event(p.trace, t, 6, globaltimer());
                bulk_commit();        // (possibly empty) group of this tile
                bulk_wait_read<0>();  // the bulk engine has read the region
                trace_event(p.trace, t, 12, globaltimer());
                if (kSG > 1) {  // regions are released in ring order
                    for (SpinGuard guard; ld_acquire_cta_smem(&s_released) != k;) {
                        guard.check("irregular in-order release");
                        __nanosleep(32);
                    }
                }
                // ring words allocated up to this tile belong to tiles stored by now
                st_release_cta_smem(&s_freed, ring_end);
                if (!in_ring) stage_release(&s_stages, meta[o].stage);
                mbar_arrive(&bar_stored[o]);
                if (kSG > 1) st_release_cta_smem(&s_released, k + 1);
            }
        }
        };
        if (kSG > 1 && sg != 0) storer_loop(std::integral_constant<uint32_t, 1>{});
        else storer_loop(std::integral_constant<uint32_t, 0>{});
        if (st == 0) {
            bulk_wait_all();  // the bulk stores are complete before the CTA exits
            trace_cta(3 + sg);
        }
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
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&lc.per_sm, kern, Layout<PART>::kThreads, kSmem)) !=
            cudaSuccess)
            return e;
        if (lc.per_sm < 1) lc.per_sm = 1;
        lc.dev = dev;
    }
    uint64_t grid = uint64_t(lc.sms) * lc.per_sm;
    if (grid > p.ntiles) grid = p.ntiles;
    p.draws = p.ntiles + uint32_t(grid);
    if (p.trace && debug_trace(size_t(p.ntiles) + grid)) p.trace_cta = p.trace + size_t(p.ntiles) * kTraceWords;
    kern<<<uint32_t(grid), Layout<PART>::kThreads, kSmem, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

size_t irregular_tile_words() { return kT; }

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
    p.pub_boards = a.pub_boards;
    p.pub_world = a.pub_world;
    p.pub_rank = a.pub_rank;
    p.pub_tag = a.pub_tag;
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
