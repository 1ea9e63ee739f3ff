// ds_regular.cu -- regular Data Sliding on sm_100a: in-place padding and
// unpadding of matrix columns (Algorithm 1; §III-A
// P:82-137; primitives §II-A P:44-48 and §IV-A).
//
// The matrix is handled as 32-bit words: an element of elem_bytes is
// elem_bytes/4 consecutive words, so a row of C elements is Cw = C*eb/4
// words.  One CTA = one OUTPUT tile of T = THREADS*ITEMS words (the paper's
// work-groups are "oblivious to number of rows and row boundaries").
// Persistent CTAs double-buffer their tiles' sources in shared memory: once
// a tile's LOADED status is published the CTA draws the next tile and
// streams its source span in through one TMA bulk copy while the current
// tile is gathered and stored.  Per tile:
//   r1 ticket + direction   pad expands (src(q) <= q): tiles in DESCENDING
//                           order; unpad shrinks (src(q) >= q): ASCENDING
//                           ("a sequential order (ascendant or descendant)",
//                           P:118)
//   r2 load sources         the contiguous span of source words of the tile's
//                           data cells, staged in shared memory with 128-bit
//                           loads (Alg. 1 first loop)
//   r3 publish LOADED +     after the tile's loads: status <- LOADED (release).
//      window wait          Then wait until every EARLIER-ticketed tile that
//                           reads sources inside this tile's output range has
//                           published LOADED.  That set is a closed-form range
//                           of tiles; the paper waits on the
//                           previous WG only (Fig. 3), a
//                           serial chain that is latency-bound on B200.
//   r4 gather + fill        output word q of row r, column c takes source
//                           r*Cw + c (c < Cw) or the fill word (pad, R1/R2)
//   r5 store                aligned 128-bit stores of the tile (Alg. 1 second
//                           loop)
// Deadlock freedom: waits only target lower tickets.
#include "ds_device.cuh"
#include "ds_internal.h"

namespace ds {
namespace {

constexpr int64_t kNoTile = -1;

struct RegParams {
    uint32_t* abase;  // 16-byte-aligned base; virtual word 0
    uint64_t mis;     // ptr - abase in words
    uint64_t out_words, in_words;  // in_words: physical end of the sources (src0 + rows*Cw)
    int64_t src0;     // slide: source of output word q is src0 + q (unpad geometry, Cw == NCw)
    uint32_t Cw, NCw;
    FastDiv div_nc;
    FastDiv64 div_nc64, div_c64;
    uint32_t fill[4];
    uint32_t wmask;   // words_per_elem - 1
    uint32_t ntiles;
    uint32_t draws;   // ntiles + gridDim.x
    uint64_t* status;
    uint64_t* ctrl;
    uint64_t* trace;  // diagnostics: per-tile events, or null
};

struct TileGeom {
    int64_t k;            // tile index (kNoTile: none)
    int64_t q0, q1;       // output words [q0, q1) of this tile
    int64_t row0;         // row of q0
    int64_t slo;          // first source word (input index) of the tile's data cells
    int64_t span;         // number of source words [slo, slo+span)
    int64_t sb;           // 16-byte aligned virtual start of the staged span
    int64_t win_lo, win_hi;  // tiles to wait for (inclusive); empty if lo > hi
    uint32_t col0;        // column (word) of q0
    int32_t base_rel;     // row0*Cw - slo
    int32_t fast;         // staged span fits in shared memory
    uint32_t bytes;       // bulk copy size (fast path)
};

// Closed-form tile geometry.  Only 64-bit divisions by the
// two row lengths, done with multiply-high (FastDiv64).
template <bool PAD, int T, int STAGE>
__device__ void tile_geometry(const RegParams& p, int64_t k, TileGeom& g) {
    const int64_t Cw = p.Cw, NCw = p.NCw, mis = int64_t(p.mis);
    const int64_t V0 = k * T;
    g.k = k;
    g.q0 = V0 - mis > 0 ? V0 - mis : 0;
    g.q1 = V0 + T - mis < int64_t(p.out_words) ? V0 + T - mis : int64_t(p.out_words);
    g.row0 = int64_t(fastdiv64(uint64_t(g.q0), p.div_nc64));
    g.col0 = uint32_t(g.q0 - g.row0 * NCw);
    const int64_t last = g.q1 - 1;
    const int64_t row1 = int64_t(fastdiv64(uint64_t(last), p.div_nc64));
    const int64_t col1 = last - row1 * NCw;
    int64_t slo, shi;
    if (PAD) {
        slo = g.col0 < Cw ? g.row0 * Cw + g.col0 : (g.row0 + 1) * Cw;
        shi = col1 < Cw ? row1 * Cw + col1 : row1 * Cw + Cw - 1;
    } else {
        slo = p.src0 + g.row0 * Cw + g.col0;
        shi = p.src0 + row1 * Cw + col1;
    }
    g.slo = slo;
    g.span = shi >= slo ? shi - slo + 1 : 0;
    g.sb = (slo + mis) & ~int64_t(3);  // lead words: inside the 16-byte chunk holding slo
    const int64_t se = (slo + mis + g.span + 3) & ~int64_t(3);
    // The bulk copy covers whole 16-byte chunks; a chunk that would pass the end
    // of the caller's buffer (pad: rows*new_cols, else the sources) is not read:
    // such a tile (at most the last one or two) takes the exact word gather.
    const int64_t buf_end = (PAD ? int64_t(p.out_words) : int64_t(p.in_words)) + mis;
    g.fast = (se - g.sb) <= STAGE && se <= buf_end;
    g.bytes = g.span > 0 && g.fast ? uint32_t(se - g.sb) * 4u : 0u;
    g.base_rel = int32_t(p.src0 + g.row0 * Cw - slo);

    // Sources physically inside this tile's output range: input words [P0, P1)
    // (source indices; a slide's sources start at physical word src0).
    const int64_t P0 = g.q0 - p.src0 > 0 ? g.q0 - p.src0 : 0;
    const int64_t P1 = (g.q1 < int64_t(p.in_words) ? g.q1 : int64_t(p.in_words)) - p.src0;
    g.win_lo = 1;
    g.win_hi = 0;
    if (P0 < P1) {
        const int64_t r = int64_t(fastdiv64(uint64_t(P0), p.div_c64)), c = P0 - r * Cw;
        const int64_t r2 = int64_t(fastdiv64(uint64_t(P1 - 1), p.div_c64)), c2 = (P1 - 1) - r2 * Cw;
        if (PAD) {  // every input word is kept; out(p) = p + row(p)*(NCw-Cw) >= p
            const int64_t olo = P0 + r * (NCw - Cw);
            const int64_t ohi = (P1 - 1) + r2 * (NCw - Cw);
            const int64_t wl = (olo + mis) / T, wh = (ohi + mis) / T;
            g.win_lo = wl > k + 1 ? wl : k + 1;
            g.win_hi = wh;
        } else {    // only columns < NCw are read; out(p) = row*NCw + col <= p
            // first / last kept source word in [P0, P1) and their outputs
            const int64_t pf = c < NCw ? P0 : (r + 1) * Cw;
            const int64_t pl = c2 < NCw ? P1 - 1 : r2 * Cw + NCw - 1;
            if (pf <= pl) {
                const int64_t of = c < NCw ? r * NCw + c : (r + 1) * NCw;
                const int64_t ol = c2 < NCw ? r2 * NCw + c2 : r2 * NCw + NCw - 1;
                const int64_t wl = (of + mis) / T, wh = (ol + mis) / T;
                g.win_lo = wl;
                g.win_hi = wh < k - 1 ? wh : k - 1;
            }
        }
    }
}

// Fill word of word-column col (elements of elem_bytes/4 words; R2).
__device__ __forceinline__ uint32_t fill_word(const RegParams& p, uint32_t col) {
    const uint32_t j = col & p.wmask;
    const uint32_t lo = (j & 1) ? p.fill[1] : p.fill[0];
    const uint32_t hi = (j & 1) ? p.fill[3] : p.fill[2];
    return (j & 2) ? hi : lo;
}

// r3: warp 0 waits until tiles [lo, hi] have published LOADED in this epoch.
__device__ __forceinline__ void wait_loaded(const uint64_t* __restrict__ status, int64_t lo,
                                            int64_t hi, uint32_t epoch, int lane) {
    for (int64_t base = lo; base <= hi; base += 32) {
        const int64_t idx = base + lane;
        bool ok = idx > hi || status_current(ld_relaxed_gpu(status_ptr(status, idx)), epoch);
        uint32_t ns = 32;
        SpinGuard guard;
        while (!__all_sync(0xffffffffu, ok)) {
            guard.check("regular window wait");
            __nanosleep(ns);
            ns = ns < 512 ? ns * 2 : 512;
            if (!ok) ok = status_current(ld_relaxed_gpu(status_ptr(status, idx)), epoch);
        }
    }
    lookback_acquire();
    __syncwarp();
}

#ifndef DS_REG_CONSUMER_WARPS
#define DS_REG_CONSUMER_WARPS 16
#endif
#ifndef DS_REG_STAGES
#define DS_REG_STAGES 3
#endif
constexpr int kConsumerWarps = DS_REG_CONSUMER_WARPS;
constexpr int kCT = 32 * kConsumerWarps;  // consumer threads
#ifndef DS_REG_TILE
#define DS_REG_TILE 8192
#endif
constexpr int kItems = DS_REG_TILE / kCT; // output words per consumer thread
constexpr int kVec = kItems / 4;
constexpr int kT = kCT * kItems;          // output words per tile (8192 = 32 KB)
static_assert(kItems % 4 == 0, "whole 128-bit vectors per consumer thread");
constexpr int kStageWords = kT + 512;     // staged source span cap (words)
constexpr int kStages = DS_REG_STAGES;
constexpr int kThreads = 32 * (2 + kConsumerWarps);  // producer, publisher, consumers
constexpr size_t kSmem = size_t(kStages) * kStageWords * 4;

struct StageMeta {
    TileGeom g;
    uint32_t epoch;
};

// Producer, slow path (the source span does not fit a stage: unpad dropping
// many columns of short rows): the warp gathers the tile's source words
// directly, stored in OUTPUT order.
template <bool PAD>
__device__ void gather_slow(const RegParams& p, const TileGeom& g, uint32_t* stage, int lane) {
    const int64_t mis = int64_t(p.mis);
    const uint32_t cnt = uint32_t(g.q1 - g.q0);
    for (uint32_t x0 = 0; x0 < cnt; x0 += 32 * 8) {
        uint32_t val[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const uint32_t x = x0 + 32 * u + lane;
            val[u] = 0;
            if (x < cnt) {
                const uint32_t t = g.col0 + x;
                const uint32_t dr = fastdiv(t, p.div_nc);
                const uint32_t col = t - dr * p.NCw;
                if (PAD && col >= p.Cw) val[u] = fill_word(p, col);
                else val[u] = ldg_stream(p.abase + p.src0 + (g.row0 + dr) * int64_t(p.Cw) + col + mis);
            }
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const uint32_t x = x0 + 32 * u + lane;
            if (x < cnt) stage[x] = val[u];
        }
    }
    __syncwarp();
}

template <bool PAD>
__global__ void __launch_bounds__(kThreads, 2) regular_kernel(const RegParams p) {
    extern __shared__ __align__(128) uint32_t smem[];
    __shared__ __align__(8) uint64_t bar_full[kStages], bar_loaded[kStages], bar_empty[kStages];
    __shared__ StageMeta meta[kStages];

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // The first ticket's atomic is in flight while thread 0 sets up the barriers.
    unsigned long long first_old = 0;
    if (tid == 0) first_old = issue_ticket(p.ctrl);
    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&bar_full[s], 32);  // every producer lane arrives (its stage writes, slow path)
            mbar_init(&bar_loaded[s], 1);
            mbar_init(&bar_empty[s], kConsumerWarps);
        }
        mbar_fence_init();
    }
    __syncthreads();
    const int64_t mis = int64_t(p.mis);

    if (warp == 0) {
        // ------------------------------------------------ producer warp
        // r1 draw + geometry, r2 start the tile's source copy; up to kStages
        // copies in flight (the publisher warp waits for them).
        for (uint32_t k = 0;; ++k) {
            const int s = k % kStages;
            const uint32_t use = k / kStages;
            uint32_t* stage = smem + s * kStageWords;
            mbar_wait(&bar_empty[s], (use & 1) ^ 1);  // consumers released tile k - kStages
            uint32_t t = 0, epoch = 0;
            if (lane == 0) {
                if (k == 0) take_ticket(p.ctrl, p.draws, first_old, t, epoch);
                else draw_ticket(p.ctrl, p.draws, t, epoch);
            }
            t = __shfl_sync(0xffffffffu, t, 0);
            epoch = __shfl_sync(0xffffffffu, epoch, 0);
            if (t >= p.ntiles) {  // one failed draw per CTA ends its work
                if (lane == 0) meta[s].g.k = kNoTile;
                __syncwarp();
                mbar_arrive(&bar_full[s]);
                break;
            }
            const int64_t kt = PAD ? int64_t(p.ntiles) - 1 - t : int64_t(t);
            if (lane == 0) {
                trace_event(p.trace, uint64_t(kt), 0, globaltimer());
                trace_event(p.trace, uint64_t(kt), 7, smid());
                debug_delay(uint64_t(kt), 0);
                tile_geometry<PAD, kT, kStageWords>(p, kt, meta[s].g);
                meta[s].epoch = epoch;
                if (meta[s].g.bytes) {
                    fence_proxy_async_smem();
                    mbar_arrive_expect_tx(&bar_full[s], meta[s].g.bytes);
                    bulk_g2s(stage, p.abase + meta[s].g.sb, meta[s].g.bytes, &bar_full[s]);
                }
            }
            __syncwarp();
            const TileGeom& g = meta[s].g;
            if (!g.bytes) {
                // slow path, or no sources at all (all fill): every lane arrives
                // after its own stage writes (so each write is ordered before the
                // phase completes, without relying on the warp barrier)
                if (g.span > 0) gather_slow<PAD>(p, g, stage, lane);
                mbar_arrive(&bar_full[s]);
            } else if (lane != 0) {
                mbar_arrive(&bar_full[s]);  // lane 0 arrived with the copy's byte count
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------ publisher warp
        // r3a: publish LOADED as soon as each tile's sources landed, in order.
        for (uint32_t k = 0;; ++k) {
            const int s = k % kStages;
            const uint32_t use = k / kStages;
            mbar_wait(&bar_full[s], use & 1);
            const int64_t kt = meta[s].g.k;
            if (lane == 0) {
                if (kt != kNoTile) {
                    trace_event(p.trace, uint64_t(kt), 1, globaltimer());
                    debug_delay(uint64_t(kt), 1);
                    publish_status(status_ptr(p.status, kt), make_status(kStateLoaded, meta[s].epoch, 0));
                    trace_event(p.trace, uint64_t(kt), 2, globaltimer());
                }
                mbar_arrive(&bar_loaded[s]);
            }
            if (kt == kNoTile) break;
        }
    } else {
        // ------------------------------------------------ consumer warps
        const int ct = tid - 64;
        for (uint32_t k = 0;; ++k) {
            const int s = k % kStages;
            const uint32_t use = k / kStages;
            const uint32_t* stage = smem + s * kStageWords;
            mbar_wait(&bar_loaded[s], use & 1);
            const TileGeom g = meta[s].g;
            if (g.k == kNoTile) break;
            const int64_t V0 = g.k * kT;

            // r3b: the first consumer warp waits for the earlier-ticketed tiles
            // whose sources lie in this tile's output range ...
            if (warp == 2) {
                if (lane == 0) trace_event(p.trace, uint64_t(g.k), 3, globaltimer());
                if (g.win_lo <= g.win_hi) wait_loaded(p.status, g.win_lo, g.win_hi, meta[s].epoch, lane);
                if (lane == 0) trace_event(p.trace, uint64_t(g.k), 4, globaltimer());
            }

            // ... while every consumer gathers its outputs (r4).
            uint32_t o[kVec][4];
            const int32_t soff = int32_t(g.slo + mis - g.sb);
            const uint32_t data_cols = PAD ? p.Cw : p.NCw;  // columns that carry source words
#pragma unroll
            for (int i = 0; i < kVec; ++i) {
                const int64_t vq = V0 + 4 * int64_t(i * kCT + ct) - mis;  // output word of slot 0
                const int64_t xq = vq - g.q0;
                uint32_t t = uint32_t(xq) + g.col0;  // only meaningful when vq >= q0
                uint32_t dr = fastdiv(t, p.div_nc);
                uint32_t col = t - dr * p.NCw;
                const bool whole = vq >= g.q0 && vq + 4 <= g.q1;
                if (whole && g.bytes && col + 4 <= data_cols) {
                    // Fast path: four data words of one row segment = four consecutive
                    // staged source words; two aligned 16-byte shared loads and a
                    // funnel shift by the segment's phase.
                    const int32_t sidx = g.base_rel + int32_t(dr * p.Cw + col) + soff;
                    const uint32_t ph = uint32_t(sidx) & 3u;
                    const u32x4 A = *reinterpret_cast<const u32x4*>(stage + (sidx & ~3));
                    const u32x4 B = ph ? *reinterpret_cast<const u32x4*>(stage + (sidx & ~3) + 4) : A;
                    const bool b0 = ph & 1u, b1 = ph & 2u;
                    const uint32_t h0 = b0 ? A.y : A.x, h1 = b0 ? A.z : A.y, h2 = b0 ? A.w : A.z;
                    const uint32_t h3 = b0 ? B.x : A.w, h4 = b0 ? B.y : B.x, h5 = b0 ? B.z : B.y;
                    o[i][0] = b1 ? h2 : h0;
                    o[i][1] = b1 ? h3 : h1;
                    o[i][2] = b1 ? h4 : h2;
                    o[i][3] = b1 ? h5 : h3;
                    continue;
                }
                if (PAD && whole && col >= p.Cw && col + 4 <= p.NCw) {  // four fill cells
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk) o[i][kk] = fill_word(p, col + kk);
                    continue;
                }
#pragma unroll
                for (int kk = 0; kk < 4; ++kk) {
                    const int64_t q = vq + kk;
                    uint32_t val = 0;
                    if (q >= g.q0 && q < g.q1) {
                        if (q == g.q0 && xq < 0) {  // tile 0 with a misaligned ptr
                            dr = 0;
                            col = g.col0;
                        }
                        if (!g.bytes && g.span > 0) {
                            val = stage[uint32_t(q - g.q0)];  // slow path: output order
                        } else if (PAD && col >= p.Cw) {
                            val = fill_word(p, col);
                        } else {
                            const int32_t srel = g.base_rel + int32_t(dr * p.Cw + col);
                            val = stage[srel + soff];
                        }
                    }
                    o[i][kk] = val;
                    if (++col == p.NCw) {
                        col = 0;
                        ++dr;
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&bar_empty[s]);  // this warp is done with the stage
            if (ct == 0) debug_delay(uint64_t(g.k), 2);
            named_bar_sync(1, kCT);  // the window wait (acquire fence) precedes every store
            if (ct == 0) trace_event(p.trace, uint64_t(g.k), 5, globaltimer());

            // r5: store stage.
#pragma unroll
            for (int i = 0; i < kVec; ++i) {
                const int64_t u = V0 + 4 * int64_t(i * kCT + ct);  // virtual
                const int64_t q = u - mis;
                if (q >= 0 && q + 4 <= int64_t(p.out_words)) {
                    stg_stream_v4(p.abase + u, o[i][0], o[i][1], o[i][2], o[i][3]);
                } else {
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk)
                        if (q + kk >= 0 && q + kk < int64_t(p.out_words))
                            stg_stream(p.abase + u + kk, o[i][kk]);
                }
            }
            if (ct == 0) trace_event(p.trace, uint64_t(g.k), 6, globaltimer());
        }
    }
}

struct LaunchCache {
    int dev = -1, sms = 0, per_sm = 0;
};

template <bool PAD>
cudaError_t launch_dir(RegParams p, cudaStream_t s) {
    static thread_local LaunchCache lc;
    auto kern = regular_kernel<PAD>;
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

size_t regular_tile_words() { return kT; }

size_t regular_tiles(const RegArgs& a) {
    const uint64_t mis = (reinterpret_cast<uintptr_t>(a.ptr) >> 2) & 3u;
    const uint64_t out_words = a.out_words_w ? a.out_words_w : a.rows * a.new_cols_w;
    return size_t((out_words + mis + kT - 1) / kT);
}

cudaError_t launch_regular(const RegArgs& a, Workspace& ws, cudaStream_t s) {
    RegParams p{};
    const uint64_t mis = (reinterpret_cast<uintptr_t>(a.ptr) >> 2) & 3u;
    p.abase = a.ptr - mis;
    p.mis = mis;
    p.out_words = a.out_words_w ? a.out_words_w : a.rows * a.new_cols_w;
    p.src0 = int64_t(a.src0_w);
    p.in_words = a.out_words_w ? a.src0_w + a.out_words_w : a.rows * a.cols_w;
    p.Cw = uint32_t(a.cols_w);
    p.NCw = uint32_t(a.new_cols_w);
    p.div_nc = make_fastdiv(p.NCw);
    p.div_nc64 = make_fastdiv64(p.NCw);
    p.div_c64 = make_fastdiv64(p.Cw ? p.Cw : 1);
    for (int i = 0; i < 4; ++i) p.fill[i] = a.fill[i];
    p.wmask = a.words_per_elem - 1;
    p.ntiles = uint32_t(regular_tiles(a));
    p.status = ws.status;
    p.ctrl = ws.ctrl;
    p.trace = debug_trace(p.ntiles);
    count_launch();
    return a.pad ? launch_dir<true>(p, s) : launch_dir<false>(p, s);
}

}  // namespace ds
