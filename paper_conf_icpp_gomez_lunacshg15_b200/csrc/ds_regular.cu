// ds_regular.cu -- regular Data Sliding on sm_100a: in-place padding and
// unpadding of matrix columns (Algorithm 1; §III-A
// P:82-137; primitives §II-A P:44-48 and §IV-A).
//
// The matrix is handled as 32-bit words: an element of elem_bytes is
// elem_bytes/4 consecutive words, so a row of C elements is Cw = C*eb/4
// words.  One CTA = one OUTPUT tile of T = THREADS*ITEMS words (the paper's
// work-groups are "oblivious to number of rows and row boundaries"):
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

struct RegParams {
    uint32_t* abase;  // 16-byte-aligned base; virtual word 0
    uint64_t mis;     // ptr - abase in words
    uint64_t out_words, in_words;
    uint32_t Cw, NCw;
    FastDiv div_nc;
    uint32_t fill[4];
    uint32_t wmask;   // words_per_elem - 1
    uint32_t ntiles;
    uint64_t* status;
    uint64_t* ctrl;
};

struct TileGeom {
    int64_t q0, q1;       // output words [q0, q1) of this tile
    int64_t row0;         // row of q0
    uint32_t col0;        // column (word) of q0
    int64_t slo;          // first source word (input index) of the tile's data cells
    int64_t span;         // number of source words [slo, slo+span)
    int64_t sb;           // 16-byte aligned virtual start of the staged span
    int64_t win_lo, win_hi;  // tiles to wait for (inclusive); empty if lo > hi
    int32_t base_rel;     // row0*Cw - slo
    int32_t fast;         // staged span fits in shared memory
};

template <bool PAD, int T, int SPAN_CAP>
__device__ void tile_geometry(const RegParams& p, int64_t k, TileGeom& g) {
    const int64_t Cw = p.Cw, NCw = p.NCw, mis = int64_t(p.mis);
    const int64_t V0 = k * T;
    g.q0 = V0 - mis > 0 ? V0 - mis : 0;
    g.q1 = V0 + T - mis < int64_t(p.out_words) ? V0 + T - mis : int64_t(p.out_words);
    g.row0 = g.q0 / NCw;
    g.col0 = uint32_t(g.q0 - g.row0 * NCw);
    const int64_t last = g.q1 - 1;
    const int64_t row1 = last / NCw;
    const int64_t col1 = last - row1 * NCw;
    int64_t slo, shi;
    if (PAD) {
        slo = g.col0 < Cw ? g.row0 * Cw + g.col0 : (g.row0 + 1) * Cw;
        shi = col1 < Cw ? row1 * Cw + col1 : row1 * Cw + Cw - 1;
    } else {
        slo = g.row0 * Cw + g.col0;
        shi = row1 * Cw + col1;
    }
    g.slo = slo;
    g.span = shi >= slo ? shi - slo + 1 : 0;
    g.sb = (slo + mis) & ~int64_t(3);
    g.fast = (slo + mis + g.span - g.sb) <= SPAN_CAP;
    g.base_rel = int32_t(g.row0 * Cw - slo);

    // Sources physically inside this tile's output range: input words [P0, P1).
    const int64_t P0 = g.q0;
    const int64_t P1 = g.q1 < int64_t(p.in_words) ? g.q1 : int64_t(p.in_words);
    g.win_lo = 1;
    g.win_hi = 0;
    if (P0 < P1) {
        if (PAD) {  // every input word is kept; out(p) = p + row(p)*(NCw-Cw) >= p
            const int64_t olo = P0 + (P0 / Cw) * (NCw - Cw);
            const int64_t ohi = (P1 - 1) + ((P1 - 1) / Cw) * (NCw - Cw);
            const int64_t wl = (olo + mis) / T, wh = (ohi + mis) / T;
            g.win_lo = wl > k + 1 ? wl : k + 1;
            g.win_hi = wh;
        } else {    // only columns < NCw are read; out(p) = row*NCw + col <= p
            const int64_t r = P0 / Cw, c = P0 - r * Cw;
            const int64_t r2 = (P1 - 1) / Cw, c2 = (P1 - 1) - r2 * Cw;
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
        bool ok = idx > hi || status_current(ld_relaxed_gpu(status + idx), epoch);
        uint32_t ns = 8;
        while (!__all_sync(0xffffffffu, ok)) {
            __nanosleep(ns);
            ns = ns < 256 ? ns * 2 : 256;
            if (!ok) ok = status_current(ld_relaxed_gpu(status + idx), epoch);
        }
    }
    fence_acq_rel_gpu();
    __syncwarp();
}

template <int THREADS, int ITEMS, bool PAD>
__global__ void __launch_bounds__(THREADS) regular_kernel(const RegParams p) {
    constexpr int VEC = ITEMS / 4;
    constexpr int T = THREADS * ITEMS;
    constexpr int SPAN_CAP = T + 512;
    constexpr int LOAD_ITERS = (SPAN_CAP / 4 + THREADS - 1) / THREADS;

    __shared__ alignas(16) uint32_t s_src[SPAN_CAP];
    __shared__ TileGeom s_g;
    __shared__ uint32_t s_epoch;
    __shared__ int64_t s_k;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {  // r1
        uint32_t t, e;
        draw_ticket(p.ctrl, p.ntiles, t, e);
        const int64_t k = PAD ? int64_t(p.ntiles) - 1 - t : int64_t(t);
        s_k = k;
        s_epoch = e;
        tile_geometry<PAD, T, SPAN_CAP>(p, k, s_g);
        debug_delay(uint64_t(k), 0);
    }
    __syncthreads();
    const int64_t k = s_k;
    const uint32_t epoch = s_epoch;
    const TileGeom g = s_g;
    const int64_t mis = int64_t(p.mis);
    const int64_t V0 = k * T;

    // r2: load stage.
    if (g.span > 0) {
        const int64_t vlo = g.slo + mis, vhi = g.slo + mis + g.span;  // virtual [vlo, vhi)
        if (g.fast) {
            u32x4 r[LOAD_ITERS];
#pragma unroll
            for (int it = 0; it < LOAD_ITERS; ++it) {
                const int64_t u = g.sb + 4 * int64_t(it * THREADS + tid);
                if (u >= vlo && u + 4 <= vhi) {
                    r[it] = ldg_stream_v4(p.abase + u);
                } else if (u < vhi) {
                    uint32_t w[4];
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk) {
                        const int64_t e = u + kk;
                        w[kk] = (e >= vlo && e < vhi) ? ldg_stream(p.abase + e) : 0u;
                    }
                    r[it] = u32x4{w[0], w[1], w[2], w[3]};
                }
            }
#pragma unroll
            for (int it = 0; it < LOAD_ITERS; ++it) {
                const int64_t u = g.sb + 4 * int64_t(it * THREADS + tid);
                if (u < vhi) *reinterpret_cast<u32x4*>(s_src + 4 * (it * THREADS + tid)) = r[it];
            }
        } else {
            // Span too long for shared memory (unpad dropping many columns of
            // short rows): gather the tile's source words directly, staged in
            // output order.
#pragma unroll
            for (int i = 0; i < VEC; ++i) {
#pragma unroll
                for (int kk = 0; kk < 4; ++kk) {
                    const int64_t q = V0 + 4 * int64_t(i * THREADS + tid) + kk - mis;
                    if (q < g.q0 || q >= g.q1) continue;
                    const uint32_t x = uint32_t(q - g.q0);
                    const uint32_t t = g.col0 + x;
                    const uint32_t dr = fastdiv(t, p.div_nc);
                    const uint32_t col = t - dr * p.NCw;
                    uint32_t val;
                    if (PAD && col >= p.Cw) val = fill_word(p, col);
                    else val = ldg_stream(p.abase + (g.row0 + dr) * int64_t(p.Cw) + col + mis);
                    s_src[x] = val;
                }
            }
        }
    }
    __syncthreads();  // the tile's loads are performed (values are in smem)
    if (tid == 0) {
        debug_delay(uint64_t(k), 1);
        st_release_gpu(p.status + k, make_status(kStateLoaded, epoch, 0));
    }

    // r3 (warp 0) overlapped with r4 (all warps).
    if (warp == 0 && g.win_lo <= g.win_hi) wait_loaded(p.status, g.win_lo, g.win_hi, epoch, lane);

    uint32_t o[VEC][4];
    const int32_t soff = int32_t(g.slo + mis - g.sb);
#pragma unroll
    for (int i = 0; i < VEC; ++i) {
        const int64_t vq = V0 + 4 * int64_t(i * THREADS + tid) - mis;  // output word of slot 0
        const int64_t xq = vq - g.q0;
        uint32_t t = uint32_t(xq) + g.col0;  // only meaningful when vq >= q0
        uint32_t dr = fastdiv(t, p.div_nc);
        uint32_t col = t - dr * p.NCw;
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
            const int64_t q = vq + kk;
            uint32_t val = 0;
            if (q >= g.q0 && q < g.q1) {
                if (q == g.q0 && xq < 0) {  // tile 0 with a misaligned ptr
                    dr = 0;
                    col = g.col0;
                }
                if (!g.fast && g.span > 0) {
                    val = s_src[uint32_t(q - g.q0)];
                } else if (PAD && col >= p.Cw) {
                    val = fill_word(p, col);
                } else {
                    const int32_t srel = g.base_rel + int32_t(dr * p.Cw + col);
                    val = s_src[srel + soff];
                }
            }
            o[i][kk] = val;
            if (++col == p.NCw) {
                col = 0;
                ++dr;
            }
        }
    }
    if (tid == 0) debug_delay(uint64_t(k), 2);
    __syncthreads();  // warp 0's window wait (with its acquire fence) is done

    // r5: store stage.
#pragma unroll
    for (int i = 0; i < VEC; ++i) {
        const int64_t u = V0 + 4 * int64_t(i * THREADS + tid);  // virtual
        const int64_t q = u - mis;
        if (q >= 0 && q + 4 <= int64_t(p.out_words)) {
            stg_stream_v4(p.abase + u, o[i][0], o[i][1], o[i][2], o[i][3]);
        } else {
#pragma unroll
            for (int kk = 0; kk < 4; ++kk)
                if (q + kk >= 0 && q + kk < int64_t(p.out_words)) stg_stream(p.abase + u + kk, o[i][kk]);
        }
    }
}

constexpr int kThreads = 256;
constexpr int kItems = 16;
constexpr int kTile = kThreads * kItems;

}  // namespace

size_t regular_tiles(const RegArgs& a) {
    const uint64_t mis = (reinterpret_cast<uintptr_t>(a.ptr) >> 2) & 3u;
    const uint64_t out_words = a.rows * a.new_cols_w;
    return size_t((out_words + mis + kTile - 1) / kTile);
}

cudaError_t launch_regular(const RegArgs& a, Workspace& ws, cudaStream_t s) {
    RegParams p{};
    const uint64_t mis = (reinterpret_cast<uintptr_t>(a.ptr) >> 2) & 3u;
    p.abase = a.ptr - mis;
    p.mis = mis;
    p.out_words = a.rows * a.new_cols_w;
    p.in_words = a.rows * a.cols_w;
    p.Cw = uint32_t(a.cols_w);
    p.NCw = uint32_t(a.new_cols_w);
    p.div_nc = make_fastdiv(p.NCw);
    for (int i = 0; i < 4; ++i) p.fill[i] = a.fill[i];
    p.wmask = a.words_per_elem - 1;
    p.ntiles = uint32_t(regular_tiles(a));
    p.status = ws.status;
    p.ctrl = ws.ctrl;
    count_launch();
    if (a.pad) regular_kernel<kThreads, kItems, true><<<p.ntiles, kThreads, 0, s>>>(p);
    else regular_kernel<kThreads, kItems, false><<<p.ntiles, kThreads, 0, s>>>(p);
    return cudaGetLastError();
}

}  // namespace ds
