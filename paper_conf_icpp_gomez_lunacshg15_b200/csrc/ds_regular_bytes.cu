// ds_regular_bytes.cu -- regular Data Sliding for 1- and 2-byte elements
// (SURVEY.md 8(f)-4): in-place padding / unpadding of matrix rows whose byte
// lengths need not be multiples of 4 (Algorithm 1; §II-A
// P:44-48, §IV-A).  Rows whose byte lengths ARE multiples of 4 go
// to the word kernel (ds_regular.cu) instead; this kernel is the general case.
//
// Same scheme as the word kernel, in byte units: persistent CTAs take OUTPUT
// tiles of T = 32 KB in dynamic-ticket order (descending for pad, ascending
// for unpad), stage the tile's source span with one TMA bulk copy,
// publish LOADED, wait for the closed-form window of earlier-ticketed tiles
// whose sources lie in the tile's output range, gather, and store:
//   r4 gather  each consumer thread builds 16-byte output chunks; a chunk that
//              lies inside one row's data is 16 consecutive source bytes at
//              any byte phase: two aligned 16-byte shared loads, a word select
//              and four funnel shifts; a chunk inside one row's fill is the
//              fill pattern; anything else (row ends, tile ends) byte by byte
//   r5 store   aligned 128-bit stores; chunks cut by the matrix ends byte-wise
// Deadlock freedom and in-place safety as in ds_regular.cu.
#include "ds_device.cuh"
#include "ds_internal.h"

namespace ds {
namespace {

constexpr int64_t kNoTileB = -1;
#ifndef DS_REGB_CONSUMER_WARPS
#define DS_REGB_CONSUMER_WARPS 16
#endif
constexpr int kBConsumerWarps = DS_REGB_CONSUMER_WARPS;
constexpr int kBCT = 32 * kBConsumerWarps;
// Output tile size TB (bytes) is a template parameter: 32 KB tiles for large
// matrices; 16 KB tiles when the output is small (< kSmallOut), where 32 KB
// tiles leave too few tiles per CTA to fill the pipeline (1-byte pad at the C2
// shape 19.5 -> 15.4 us; at 16384 x 16384 16 KB tiles cost 15 %).
#ifndef DS_REGB_SMALL_TILE
#define DS_REGB_SMALL_TILE 16384
#endif
constexpr int kTBLarge = 32768, kTBSmall = DS_REGB_SMALL_TILE;
constexpr uint64_t kSmallOut = 64ull << 20;
template <int TB>
struct BCfg {
    static constexpr int Chunks = TB / 16 / kBCT;      // 16-byte chunks per consumer thread
    static constexpr int StageBytes = TB + 2048;       // staged source span cap
    static constexpr int StageAlloc = StageBytes + 32; // vector reads may pass the span by 16 bytes
    static_assert(Chunks >= 1 && Chunks * 16 * kBCT == TB, "tile size");
    static_assert(StageBytes % 16 == 0 && StageAlloc % 16 == 0, "stage alignment");
};
#ifndef DS_REGB_STAGES
#define DS_REGB_STAGES 3
#endif
constexpr int kBStages = DS_REGB_STAGES;
constexpr int kBThreads = 32 * (2 + kBConsumerWarps);
template <int TB>
constexpr size_t smem_b() { return size_t(kBStages) * BCfg<TB>::StageAlloc; }

struct RegBParams {
    uint8_t* abase;        // 16-byte-aligned base; virtual byte 0
    uint64_t mis;          // ptr - abase (0..15)
    uint64_t out_bytes, in_bytes;
    uint32_t Cb, NCb;      // row lengths in bytes (before / after)
    FastDiv div_nc;
    FastDiv64 div_nc64, div_c64;
    uint32_t eb;           // element bytes (1 or 2)
    uint8_t fill[2];
    uint32_t ntiles;
    uint32_t draws;
    uint64_t* status;
    uint64_t* ctrl;
    uint64_t* trace;       // diagnostics: per-tile events, or null (as the word kernel)
};

struct TileGeomB {
    int64_t k;
    int64_t q0, q1;        // output bytes [q0, q1)
    int64_t row0;
    int64_t slo, span;     // source bytes [slo, slo + span)
    int64_t sb;            // 16-byte aligned virtual start of the staged span
    int64_t win_lo, win_hi;
    uint32_t col0;
    int32_t base_rel;      // row0*Cb - slo
    uint32_t bytes;        // bulk copy size (0: slow path or nothing to load)
};

// Closed-form geometry, the word kernel's formulas in bytes.
template <bool PAD, int TB>
__device__ void tile_geometry_b(const RegBParams& p, int64_t k, TileGeomB& g) {
    constexpr int64_t kTB = TB;
    const int64_t Cb = p.Cb, NCb = p.NCb, mis = int64_t(p.mis);
    const int64_t V0 = k * kTB;
    g.k = k;
    g.q0 = V0 - mis > 0 ? V0 - mis : 0;
    g.q1 = V0 + kTB - mis < int64_t(p.out_bytes) ? V0 + kTB - mis : int64_t(p.out_bytes);
    g.row0 = int64_t(fastdiv64(uint64_t(g.q0), p.div_nc64));
    g.col0 = uint32_t(g.q0 - g.row0 * NCb);
    const int64_t last = g.q1 - 1;
    const int64_t row1 = int64_t(fastdiv64(uint64_t(last), p.div_nc64));
    const int64_t col1 = last - row1 * NCb;
    int64_t slo, shi;
    if (PAD) {
        slo = g.col0 < Cb ? g.row0 * Cb + g.col0 : (g.row0 + 1) * Cb;
        shi = col1 < Cb ? row1 * Cb + col1 : row1 * Cb + Cb - 1;
    } else {
        slo = g.row0 * Cb + g.col0;
        shi = row1 * Cb + col1;
    }
    g.slo = slo;
    g.span = shi >= slo ? shi - slo + 1 : 0;
    g.sb = (slo + mis) & ~int64_t(15);  // lead bytes: inside the 16-byte chunk holding slo
    const int64_t se = (slo + mis + g.span + 15) & ~int64_t(15);
    // whole 16-byte chunks, never past the end of the caller's buffer (pad:
    // rows*new_cols bytes, unpad: rows*cols): else the exact byte gather
    const int64_t buf_end = (PAD ? int64_t(p.out_bytes) : int64_t(p.in_bytes)) + mis;
    g.bytes = (g.span > 0 && se - g.sb <= BCfg<TB>::StageBytes && se <= buf_end) ? uint32_t(se - g.sb) : 0u;
    g.base_rel = int32_t(g.row0 * Cb - slo);

    // Earlier-ticketed tiles whose sources lie in this tile's output bytes.
    const int64_t P0 = g.q0;
    const int64_t P1 = g.q1 < int64_t(p.in_bytes) ? g.q1 : int64_t(p.in_bytes);
    g.win_lo = 1;
    g.win_hi = 0;
    if (P0 < P1) {
        const int64_t r = int64_t(fastdiv64(uint64_t(P0), p.div_c64)), c = P0 - r * Cb;
        const int64_t r2 = int64_t(fastdiv64(uint64_t(P1 - 1), p.div_c64)), c2 = (P1 - 1) - r2 * Cb;
        if (PAD) {
            const int64_t olo = P0 + r * (NCb - Cb);
            const int64_t ohi = (P1 - 1) + r2 * (NCb - Cb);
            const int64_t wl = (olo + mis) / kTB, wh = (ohi + mis) / kTB;
            g.win_lo = wl > k + 1 ? wl : k + 1;
            g.win_hi = wh;
        } else {
            const int64_t pf = c < NCb ? P0 : (r + 1) * Cb;
            const int64_t pl = c2 < NCb ? P1 - 1 : r2 * Cb + NCb - 1;
            if (pf <= pl) {
                const int64_t of = c < NCb ? r * NCb + c : (r + 1) * NCb;
                const int64_t ol = c2 < NCb ? r2 * NCb + c2 : r2 * NCb + NCb - 1;
                const int64_t wl = (of + mis) / kTB, wh = (ol + mis) / kTB;
                g.win_lo = wl;
                g.win_hi = wh < k - 1 ? wh : k - 1;
            }
        }
    }
}

__device__ __forceinline__ void wait_loaded_b(const uint64_t* __restrict__ status, int64_t lo, int64_t hi,
                                              uint32_t epoch, int lane) {
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

// 16 consecutive bytes of the stage starting at byte offset sidx (any phase):
// two aligned 16-byte shared loads, a word select and four funnel shifts.
// Reads up to 31 bytes past sidx (inside the stage allocation's slack).
__device__ __forceinline__ void load16(const uint32_t* stage32, int32_t sidx, uint32_t out[4]) {
    const int32_t w = sidx >> 2;
    const uint32_t bph = uint32_t(sidx) & 3u, wph = uint32_t(w) & 3u;
    const u32x4 A = *reinterpret_cast<const u32x4*>(stage32 + (w & ~3));
    const u32x4 B = *reinterpret_cast<const u32x4*>(stage32 + (w & ~3) + 4);
    const uint32_t a[8] = {A.x, A.y, A.z, A.w, B.x, B.y, B.z, B.w};
    uint32_t h[5];
#pragma unroll
    for (int j = 0; j < 5; ++j) {
        uint32_t v = a[j];
#pragma unroll
        for (uint32_t q = 1; q < 4; ++q)
            if (wph == q) v = a[j + q];
        h[j] = v;
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) out[j] = __funnelshift_r(h[j], h[j + 1], 8 * bph);
}

__device__ __forceinline__ uint8_t ldg_u8(const uint8_t* p) {
    uint16_t v;
    asm volatile("ld.global.L1::no_allocate.u8 %0, [%1];" : "=h"(v) : "l"(p));
    return uint8_t(v);
}
__device__ __forceinline__ void stg_u8(uint8_t* p, uint8_t v) {
    asm volatile("st.global.L1::no_allocate.u8 [%0], %1;" ::"l"(p), "h"(uint16_t(v)) : "memory");
}

// Slow producer path (the span does not fit a stage): the warp gathers the
// tile's source bytes straight from global memory, in OUTPUT order.
template <bool PAD>
__device__ void gather_slow_b(const RegBParams& p, const TileGeomB& g, uint8_t* stage, int lane) {
    const uint32_t cnt = uint32_t(g.q1 - g.q0);
    for (uint32_t x = lane; x < cnt; x += 32) {
        const uint32_t t = g.col0 + x;
        const uint32_t dr = fastdiv(t, p.div_nc);
        const uint32_t col = t - dr * p.NCb;
        uint8_t v = 0;
        if (PAD && col >= p.Cb) v = p.fill[col % p.eb];
        else v = ldg_u8(p.abase + (g.row0 + dr) * int64_t(p.Cb) + col + p.mis);
        stage[x] = v;
    }
    __syncwarp();
}

template <bool PAD, int TB>
__global__ void __launch_bounds__(kBThreads, 2) regular_bytes_kernel(const RegBParams p) {
    constexpr int64_t kTB = TB;
    constexpr int kBChunks = BCfg<TB>::Chunks;
    constexpr int kBStageAlloc = BCfg<TB>::StageAlloc;
    extern __shared__ __align__(128) uint8_t smem8[];
    __shared__ __align__(8) uint64_t bar_full[kBStages], bar_loaded[kBStages], bar_empty[kBStages];
    __shared__ TileGeomB geo[kBStages];
    __shared__ uint32_t geo_epoch[kBStages];

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // The first ticket's atomic is in flight while thread 0 sets up the barriers.
    unsigned long long first_old = 0;
    if (tid == 0) first_old = issue_ticket(p.ctrl);
    if (tid == 0) {
        for (int s = 0; s < kBStages; ++s) {
            mbar_init(&bar_full[s], 32);  // every producer lane arrives (its stage writes, slow path)
            mbar_init(&bar_loaded[s], 1);
            mbar_init(&bar_empty[s], kBConsumerWarps);
        }
        mbar_fence_init();
    }
    __syncthreads();
    const int64_t mis = int64_t(p.mis);

    if (warp == 0) {
        // ---------------------------------------------- producer: r1 + r2
        for (uint32_t k = 0;; ++k) {
            const int s = k % kBStages;
            uint8_t* stage = smem8 + size_t(s) * kBStageAlloc;
            mbar_wait(&bar_empty[s], ((k / kBStages) & 1) ^ 1);
            uint32_t t = 0, epoch = 0;
            if (lane == 0) {
                if (k == 0) take_ticket(p.ctrl, p.draws, first_old, t, epoch);
                else draw_ticket(p.ctrl, p.draws, t, epoch);
            }
            t = __shfl_sync(0xffffffffu, t, 0);
            epoch = __shfl_sync(0xffffffffu, epoch, 0);
            if (t >= p.ntiles) {
                if (lane == 0) geo[s].k = kNoTileB;
                __syncwarp();
                mbar_arrive(&bar_full[s]);
                break;
            }
            const int64_t kt = PAD ? int64_t(p.ntiles) - 1 - t : int64_t(t);
            if (lane == 0) {
                debug_delay(uint64_t(kt), 0);
                trace_event(p.trace, uint64_t(kt), 0, globaltimer());
                trace_event(p.trace, uint64_t(kt), 7, smid());
                tile_geometry_b<PAD, TB>(p, kt, geo[s]);
                geo_epoch[s] = epoch;
                if (geo[s].bytes) {
                    fence_proxy_async_smem();
                    mbar_arrive_expect_tx(&bar_full[s], geo[s].bytes);
                    bulk_g2s(stage, p.abase + geo[s].sb, geo[s].bytes, &bar_full[s]);
                }
            }
            __syncwarp();
            const TileGeomB& g = geo[s];
            if (!g.bytes) {
                // every lane arrives after its own stage writes
                if (g.span > 0) gather_slow_b<PAD>(p, g, stage, lane);
                mbar_arrive(&bar_full[s]);
            } else if (lane != 0) {
                mbar_arrive(&bar_full[s]);  // lane 0 arrived with the copy's byte count
            }
        }
    } else if (warp == 1) {
        // ---------------------------------------------- publisher: LOADED
        for (uint32_t k = 0;; ++k) {
            const int s = k % kBStages;
            mbar_wait(&bar_full[s], (k / kBStages) & 1);
            const int64_t kt = geo[s].k;
            if (lane == 0) {
                if (kt != kNoTileB) {
                    trace_event(p.trace, uint64_t(kt), 1, globaltimer());
                    debug_delay(uint64_t(kt), 1);
                    publish_status(status_ptr(p.status, kt), make_status(kStateLoaded, geo_epoch[s], 0));
                    trace_event(p.trace, uint64_t(kt), 2, globaltimer());
                }
                mbar_arrive(&bar_loaded[s]);
            }
            if (kt == kNoTileB) break;
        }
    } else {
        // ---------------------------------------------- consumers: r3b, r4, r5
        const int ct = tid - 64;
        const uint32_t data_cols = PAD ? p.Cb : p.NCb;
        for (uint32_t k = 0;; ++k) {
            const int s = k % kBStages;
            const uint8_t* stage = smem8 + size_t(s) * kBStageAlloc;
            const uint32_t* stage32 = reinterpret_cast<const uint32_t*>(stage);
            mbar_wait(&bar_loaded[s], (k / kBStages) & 1);
            const TileGeomB g = geo[s];
            if (g.k == kNoTileB) break;
            if (warp == 2) {
                if (lane == 0) trace_event(p.trace, uint64_t(g.k), 3, globaltimer());
                if (g.win_lo <= g.win_hi) wait_loaded_b(p.status, g.win_lo, g.win_hi, geo_epoch[s], lane);
                if (lane == 0) trace_event(p.trace, uint64_t(g.k), 4, globaltimer());
            }
            const int64_t V0 = g.k * kTB;
            const int32_t soff = int32_t(g.slo + mis - g.sb);
            uint32_t o[kBChunks][4];
#pragma unroll
            for (int i = 0; i < kBChunks; ++i) {
                const int64_t vq = V0 + 16 * int64_t(i * kBCT + ct) - mis;  // output byte of the chunk start
                const int64_t xq = vq - g.q0;
                uint32_t t = uint32_t(xq) + g.col0;
                uint32_t dr = fastdiv(t, p.div_nc);
                uint32_t col = t - dr * p.NCb;
                const bool whole = vq >= g.q0 && vq + 16 <= g.q1;
                // fast path: the chunk lies in one output row and starts in its data;
                // for pad it may end in the row's fill (merged below)
                if (whole && g.bytes && col < data_cols && col + 16 <= (PAD ? p.NCb : data_cols)) {
                    // 16 consecutive source bytes at byte offset sidx of the stage
                    const int32_t sidx = g.base_rel + int32_t(dr * p.Cb + col) + soff;
                    load16(stage32, sidx, o[i]);
                    if (PAD && col + 16 > data_cols) {
                        // the row's last nd data bytes, then its fill: the bytes read past
                        // the data end (inside the staged span + slack) are replaced
                        const int32_t nd = int32_t(data_cols - col);
                        const uint32_t f0 = p.fill[0], f1 = p.fill[p.eb - 1];
                        uint32_t pat = (col & 1u) && p.eb == 2 ? (f1 | f0 << 8) : (f0 | f1 << 8);
                        pat |= pat << 16;
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            const int32_t keep = nd - 4 * j;
                            const uint32_t m = keep >= 4 ? 0xffffffffu : keep <= 0 ? 0u : (1u << (8 * keep)) - 1u;
                            o[i][j] = (o[i][j] & m) | (pat & ~m);
                        }
                    }
                    continue;
                }
                if (!PAD && whole && g.bytes && p.NCb >= 16 && col + 16 > p.NCb) {
                    // unpad: the end of output row r, then the start of row r + 1, whose
                    // source follows the Cb - NCb dropped bytes: two 16-byte reads, merged
                    const int32_t sidx = g.base_rel + int32_t(dr * p.Cb + col) + soff;
                    uint32_t o1[4], o2[4];
                    load16(stage32, sidx, o1);
                    load16(stage32, sidx + int32_t(p.Cb - p.NCb), o2);
                    const int32_t nd = int32_t(p.NCb - col);  // bytes of row r (1..15)
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int32_t keep = nd - 4 * j;
                        const uint32_t m = keep >= 4 ? 0xffffffffu : keep <= 0 ? 0u : (1u << (8 * keep)) - 1u;
                        o[i][j] = (o1[j] & m) | (o2[j] & ~m);
                    }
                    continue;
                }
                if (PAD && whole && col >= p.Cb && col + 16 <= p.NCb) {  // 16 fill bytes
                    const uint32_t f0 = p.fill[0], f1 = p.fill[p.eb - 1];
                    uint32_t pat = (col & 1u) && p.eb == 2 ? (f1 | f0 << 8) : (f0 | f1 << 8);
                    pat |= pat << 16;
                    o[i][0] = o[i][1] = o[i][2] = o[i][3] = pat;
                    continue;
                }
                // byte by byte (row ends, fill edges, tile / matrix ends)
                uint32_t wv[4] = {0, 0, 0, 0};
                for (int j = 0; j < 16; ++j) {
                    const int64_t q = vq + j;
                    uint32_t val = 0;
                    if (q >= g.q0 && q < g.q1) {
                        if (q == g.q0 && xq < 0) {  // tile 0 with a misaligned ptr
                            dr = 0;
                            col = g.col0;
                        }
                        if (!g.bytes && g.span > 0) val = stage[uint32_t(q - g.q0)];
                        else if (PAD && col >= p.Cb) val = p.fill[p.eb == 2 ? (col & 1u) : 0u];
                        else val = stage[g.base_rel + int32_t(dr * p.Cb + col) + soff];
                    }
                    wv[j >> 2] |= val << (8 * (j & 3));
                    if (q >= g.q0 && ++col == p.NCb) {
                        col = 0;
                        ++dr;
                    }
                }
#pragma unroll
                for (int j = 0; j < 4; ++j) o[i][j] = wv[j];
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&bar_empty[s]);
            if (ct == 0) debug_delay(uint64_t(g.k), 2);
            named_bar_sync(1, kBCT);  // the window wait precedes every store
            if (ct == 0) trace_event(p.trace, uint64_t(g.k), 5, globaltimer());
#pragma unroll
            for (int i = 0; i < kBChunks; ++i) {
                const int64_t u = V0 + 16 * int64_t(i * kBCT + ct);  // virtual byte
                const int64_t q = u - mis;
                if (q >= 0 && q + 16 <= int64_t(p.out_bytes)) {
                    stg_stream_v4(reinterpret_cast<uint32_t*>(p.abase + u), o[i][0], o[i][1], o[i][2], o[i][3]);
                } else {
                    for (int j = 0; j < 16; ++j)
                        if (q + j >= 0 && q + j < int64_t(p.out_bytes))
                            stg_u8(p.abase + u + j, uint8_t(o[i][j >> 2] >> (8 * (j & 3))));
                }
            }
            if (ct == 0) trace_event(p.trace, uint64_t(g.k), 6, globaltimer());
        }
    }
}

struct LaunchCacheB {
    int dev = -1, sms = 0, per_sm = 0;
};

template <bool PAD, int TB>
cudaError_t launch_dir_b(RegBParams p, cudaStream_t s) {
    constexpr size_t kBSmem = smem_b<TB>();
    static thread_local LaunchCacheB lc;
    auto kern = regular_bytes_kernel<PAD, TB>;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (lc.dev != dev) {
        if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kBSmem))) !=
            cudaSuccess)
            return e;
        if ((e = cudaDeviceGetAttribute(&lc.sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess)
            return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&lc.per_sm, kern, kBThreads, kBSmem)) !=
            cudaSuccess)
            return e;
        if (lc.per_sm < 1) lc.per_sm = 1;
        lc.dev = dev;
    }
    uint64_t grid = uint64_t(lc.sms) * lc.per_sm;
    if (grid > p.ntiles) grid = p.ntiles;
    p.draws = p.ntiles + uint32_t(grid);
    kern<<<uint32_t(grid), kBThreads, kBSmem, s>>>(p);
    return cudaGetLastError();
}

}  // namespace

size_t regular_bytes_tile_bytes() { return kTBLarge; }

// Output tile bytes a launch uses.
static int64_t tile_bytes_for(const RegBytesArgs& a) {
    return a.rows * a.new_cols_b < kSmallOut ? kTBSmall : kTBLarge;
}

size_t regular_bytes_tiles(const RegBytesArgs& a) {
    const uint64_t mis = reinterpret_cast<uintptr_t>(a.ptr) & 15u;
    const int64_t tb = tile_bytes_for(a);
    return size_t((a.rows * a.new_cols_b + mis + tb - 1) / tb);
}

cudaError_t launch_regular_bytes(const RegBytesArgs& a, Workspace& ws, cudaStream_t s) {
    RegBParams p{};
    const uint64_t mis = reinterpret_cast<uintptr_t>(a.ptr) & 15u;
    p.abase = a.ptr - mis;
    p.mis = mis;
    p.out_bytes = a.rows * a.new_cols_b;
    p.in_bytes = a.rows * a.cols_b;
    p.Cb = uint32_t(a.cols_b);
    p.NCb = uint32_t(a.new_cols_b);
    p.div_nc = make_fastdiv(p.NCb);
    p.div_nc64 = make_fastdiv64(p.NCb);
    p.div_c64 = make_fastdiv64(p.Cb ? p.Cb : 1);
    p.eb = a.elem_bytes;
    p.fill[0] = a.fill[0];
    p.fill[1] = a.fill[1];
    p.ntiles = uint32_t(regular_bytes_tiles(a));
    p.trace = debug_trace(p.ntiles);
    p.status = ws.status;
    p.ctrl = ws.ctrl;
    count_launch();
    if (tile_bytes_for(a) == kTBSmall)
        return a.pad ? launch_dir_b<true, kTBSmall>(p, s) : launch_dir_b<false, kTBSmall>(p, s);
    return a.pad ? launch_dir_b<true, kTBLarge>(p, s) : launch_dir_b<false, kTBLarge>(p, s);
}

}  // namespace ds
