// k_integral.cu -- K1: pyramid scaling fused with integral + squared-integral images.
//
// Paper: "the scaling stage generates n resized images by subsampling the decompressed
// frame ... tex2D linear interpolation"; "integral images are computed ... with a
// combination of parallel prefix sum [17][18] and matrix transposition operations [19]"
// (P:L368-384).  B200 design: no transpose is materialised.
// Each level is cut into tiles of 32 rows x 128 ii columns.  k_marg resamples a tile's pixels
// from the frame (exact integer bilinear, reading R2), writes them to a level-image scratch
// buffer (an HBM round trip of ~12 MB per 1080p frame) and its per-tile marginal sums;
// k_carry / k_corner turn the marginals into row carries, column carries and tile corners;
// k_tile re-reads the level image, runs warp-shuffle row scans, stages the row prefixes in
// shared memory and runs a coalesced, vectorised (uint4) column scan, so ii/sqii are written to
// HBM exactly once and all tiles of all levels of all frames of a group run in parallel.
// K1 serves fd_integral, the soft-cascade path (k_soft) and the round-1 split K2 schedule; the
// default detection path (f1) needs only k_level's level images (below).
#include "fd_internal.h"

namespace fdk {

// (k_marg / k_tile compiled for 6 resident CTAs per SM -- 40 registers -- measured no faster)

// ---------------------------------------------------------------- scaling (reading R2)
// The taps are addressed from one corner: (x0, y0) and (x0 + 1, y0 + 1).  Where reading R2 clamps
// x1 = x0 = W - 1 (the sample lies past the last pixel centre), the corner moves to W - 2 with
// weight a_x = 256 instead: p00 (256 - 256) + p01 * 256 = p[W-1] * 256 = p[W-1] (256 - a) + p[W-1] a,
// the same integer; likewise for rows.  So every tap is the corner address + {0, 1, pitch,
// pitch + 1} (two 64-bit addresses per pixel, immediate offsets for the rest).  Needs W, H >= 2.
struct RowSample {
    const uint8_t* r0;      // row y0 (its successor is r0 + pitch)
    int ay;
};

__device__ __forceinline__ RowSample row_sample(const uint8_t* frame, int pitch, int H, int r16, int y) {
    const long long sy = ((2LL * y + 1) * (long long)r16 - 65536) >> 1;
    const int y0 = (int)(sy >> 16);
    RowSample s;
    s.ay = y0 < H - 1 ? (int)((sy >> 8) & 255) : 256;
    s.r0 = frame + (size_t)(y0 < H - 1 ? y0 : H - 2) * pitch;
    return s;
}

struct ColSample {
    int x0, ax;
};

__device__ __forceinline__ ColSample col_sample(int W, int r16, int x) {
    const long long sx = ((2LL * x + 1) * (long long)r16 - 65536) >> 1;
    const int x0 = (int)(sx >> 16);
    ColSample c;
    c.x0 = x0 < W - 1 ? x0 : W - 2;
    c.ax = x0 < W - 1 ? (int)((sx >> 8) & 255) : 256;
    return c;
}

// p = (p00(256-ax)(256-ay) + p01 ax(256-ay) + p10(256-ax)ay + p11 ax ay + 2^15) >> 16,
// evaluated as two horizontal lerps then one vertical (identical in exact integer arithmetic).
__device__ __forceinline__ uint32_t bilinear(const RowSample& r, int pitch, const ColSample& c) {
    const uint8_t* a = r.r0 + c.x0;
    const uint8_t* b = a + pitch;
    const int p00 = __ldg(a), p01 = __ldg(a + 1);
    const int p10 = __ldg(b), p11 = __ldg(b + 1);
    const int h0 = p00 * (256 - c.ax) + p01 * c.ax;
    const int h1 = p10 * (256 - c.ax) + p11 * c.ax;
    return (uint32_t)((h0 * (256 - r.ay) + h1 * r.ay + 32768) >> 16);
}

__device__ __forceinline__ uint32_t level_pixel(const uint8_t* frame, int pitch, int srcW, int srcH, int r16,
                                                int x, int y) {
    if (r16 == 65536) return __ldg(frame + (size_t)y * pitch + x);   // level 0: identity
    const RowSample r = row_sample(frame, pitch, srcH, r16, y);
    return bilinear(r, pitch, col_sample(srcW, r16, x));
}

// The 4 level pixels of row y at columns x .. x+3 (0 at or beyond the level width).  Identity
// level: one aligned 4-byte load when the frame allows it.  Bilinear levels: branch-free -- the
// column taps cs[] are clamped into the frame (col_sample of min(x + j, W_k - 1)), every tap is
// loaded and the pixels past the level width are masked afterwards.
__device__ __forceinline__ void tile_row_pixels(const uint8_t* frame, const PlanDev& p, const LevelDev& L, int y, int x,
                                                const ColSample* cs, uint32_t* pv) {
    if (L.r16 == 65536) {
        const uint8_t* row = frame + (size_t)y * p.pitch;
        if (p.aligned4 && x + 4 <= p.pitch) {
            const uint32_t w = __ldg(reinterpret_cast<const uint32_t*>(row + x));
#pragma unroll
            for (int j = 0; j < 4; ++j) pv[j] = x + j < L.W ? (w >> (8 * j)) & 255u : 0u;
        } else {
#pragma unroll
            for (int j = 0; j < 4; ++j) pv[j] = x + j < L.W ? (uint32_t)__ldg(row + x + j) : 0u;
        }
        return;
    }
    const RowSample rs = row_sample(frame, p.pitch, p.H, L.r16, y);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const uint32_t v = bilinear(rs, p.pitch, cs[j]);
        pv[j] = x + j < L.W ? v : 0u;
    }
}

// Staged resampling (reading R2 unchanged, only where the taps come from): for levels with
// f <= 2.25 the source rows and columns that the 32 x 128 output pixels of a K1 tile sample are
// copied to shared memory with 16-byte loads, and the bilinear taps are read there with 32-bit
// addresses.  For such f every coordinate product fits 32 bits: (2 * 3840 + 1) * 2.25 * 2^16 < 2^31.
constexpr int STAGE_R16_MAX = 147456;              // 2.25 * 2^16
constexpr int SRC_ROWS = 74, SRC_PITCH = 336;      // >= 31 * 2.25 + 3 rows; >= 127 * 2.25 + 3 + 15 + 1 columns

struct SrcStage {
    int ys0, xa;                                   // first staged source row / (16-aligned) column
};

__device__ __forceinline__ int src_coord(int v, int r16, int lim, int* frac) {
    const int sv = ((2 * v + 1) * r16 - 65536) >> 1;
    *frac = (sv >> 8) & 255;
    const int v0 = sv >> 16;
    return v0 < lim - 1 ? v0 : lim - 1;
}

// Copies the tile's source region to S (all threads; ends with a barrier).  The column right of
// the last frame column is a copy of it, so the tap x0 + 1 is the clamped x1 everywhere.
__device__ __forceinline__ SrcStage stage_source(const uint8_t* __restrict__ frame, const PlanDev& p, const LevelDev& L,
                                                 int y0, int rows, int x0, uint8_t* S) {
    int fr;
    SrcStage st;
    st.ys0 = src_coord(y0, L.r16, p.H, &fr);
    const int ys1 = min(p.H - 1, src_coord(y0 + rows - 1, L.r16, p.H, &fr) + 1);
    const int xs0 = src_coord(x0, L.r16, p.W, &fr);
    const int xs1 = min(p.W - 1, src_coord(min(x0 + CHUNK, L.W) - 1, L.r16, p.W, &fr) + 1);
    st.xa = xs0 & ~15;
    const int nch = (xs1 - st.xa) / 16 + 1, nr = ys1 - st.ys0 + 1;
    for (int i = threadIdx.x; i < nr * nch; i += K1_THREADS) {
        const int r = i / nch, c = i - r * nch;
        *reinterpret_cast<uint4*>(S + r * SRC_PITCH + 16 * c) =
            __ldg(reinterpret_cast<const uint4*>(frame + (size_t)(st.ys0 + r) * p.pitch + st.xa + 16 * c));
    }
    __syncthreads();
    if (xs1 == p.W - 1)
        for (int r = threadIdx.x; r < nr; r += K1_THREADS) S[r * SRC_PITCH + p.W - st.xa] = S[r * SRC_PITCH + p.W - 1 - st.xa];
    __syncthreads();
    return st;
}

// The 4 level pixels of row y at columns x .. x+3 from the staged source (o[j]: staged column of
// x0(x + j), ax[j] its weight), 0 at or beyond the level width.
__device__ __forceinline__ void staged_row_pixels(const uint8_t* __restrict__ S, const PlanDev& p, const LevelDev& L,
                                                  const SrcStage& st, int y, int x, const int* o, const int* ax,
                                                  uint32_t* pv) {
    int ay;
    const int y0s = src_coord(y, L.r16, p.H, &ay);
    const int y1s = y0s + 1 < p.H ? y0s + 1 : p.H - 1;
    const uint8_t* r0 = S + (y0s - st.ys0) * SRC_PITCH;
    const uint8_t* r1 = S + (y1s - st.ys0) * SRC_PITCH;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const int h0 = (int)r0[o[j]] * (256 - ax[j]) + (int)r0[o[j] + 1] * ax[j];
        const int h1 = (int)r1[o[j]] * (256 - ax[j]) + (int)r1[o[j] + 1] * ax[j];
        const uint32_t v = (uint32_t)((h0 * (256 - ay) + h1 * ay + 32768) >> 16);
        pv[j] = x + j < L.W ? v : 0u;
    }
}

__device__ __forceinline__ int find_level_k1(const PlanDev& p, int t) {
    int k = 0;
    while (k + 1 < p.n_levels && p.lv[k + 1].k1t0 <= t) ++k;
    return k;
}

// ---------------------------------------------------------------- K1a: per-tile marginals
// colsum[band][plane][x] = sum over the tile's rows of p (plane 0) / p^2 (plane 1)
// rowsum[band][chunk][plane][r] = sum over the tile's columns
__global__ void __launch_bounds__(K1_THREADS) k_marg(const uint8_t* __restrict__ frames, const __grid_constant__ PlanDev p,
                                                     K1Scratch s) {
    __shared__ uint32_t red_s[8][CHUNK], red_q[8][CHUNK];
    __shared__ uint8_t raw[BAND + 2][CHUNK + 4];       // filtering stage: resampled rows with a 1-px halo
    const int g = blockIdx.y;
    const int k = find_level_k1(p, blockIdx.x);
    const LevelDev& L = p.lv[k];
    const int tl = blockIdx.x - L.k1t0;
    const int b = tl / L.nchunks, c = tl % L.nchunks;
    const int y0 = b * BAND, rows = min(BAND, L.H - y0);
    const int x0 = c * CHUNK;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint8_t* frame = frames + (size_t)g * p.H * p.pitch;
    const int x = x0 + 4 * lane;
    // (staged resampling, as in k_level, measured slower here: 14.5 vs 13.5 ms per 512 frames --
    // the extra 25 KB of shared memory costs this short-lived, latency-bound kernel occupancy)
    ColSample cs[4];
    if (L.r16 != 65536) {
#pragma unroll
        for (int j = 0; j < 4; ++j) cs[j] = col_sample(p.W, L.r16, min(x + j, L.W - 1));
    }
    uint32_t cols[4] = {0, 0, 0, 0}, colq[4] = {0, 0, 0, 0};
    uint32_t* rowsum = s.row + (size_t)g * p.row_frame + L.row_off + (size_t)(b * L.nchunks + c) * 2 * BAND;
    uint8_t* lvl = s.lvl + (size_t)g * p.lvl_frame + L.lvl_off;
    if (p.filter) {
        // f2 filtering stage (reading R3b): the resampled level at rows y0-1 .. y0+rows and columns
        // x0-1 .. x0+CHUNK, clamped to the level (clamp-to-edge), then the 3x3 binomial below
        for (int r = warp; r < rows + 2; r += K1_THREADS / 32) {
            const int yy = min(max(y0 - 1 + r, 0), L.H - 1);
            for (int q = lane; q < CHUNK + 2; q += 32) {
                const int xx = min(max(x0 - 1 + q, 0), L.W - 1);
                raw[r][q] = (uint8_t)level_pixel(frame, p.pitch, p.W, p.H, L.r16, xx, yy);
            }
        }
        __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < BAND / 8; ++i) {
        const int r = warp + 8 * i;
        if (r < rows) {
            uint32_t pv[4];
            if (p.filter) {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int q = x + j - x0 + 1;            // raw column of pixel x + j
                    uint32_t v = 0;
                    if (x + j < L.W) {
#pragma unroll
                        for (int dy = 0; dy < 3; ++dy) {
                            const uint32_t h = raw[r + dy][q - 1] + 2u * raw[r + dy][q] + raw[r + dy][q + 1];
                            v += (dy == 1 ? 2u : 1u) * h;
                        }
                        v = (v + 8u) >> 4;
                    }
                    pv[j] = v;
                }
            } else {
                tile_row_pixels(frame, p, L, y0 + r, x, cs, pv);
            }
            if (x < L.PB)      // level image row (pitch PB), 4 pixels per lane as one aligned word (0 past W)
                *reinterpret_cast<uint32_t*>(lvl + (size_t)(y0 + r) * L.PB + x) =
                    pv[0] | (pv[1] << 8) | (pv[2] << 16) | (pv[3] << 24);
            uint32_t rs = 0, rq = 0;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const uint32_t q = pv[j] * pv[j];
                rs += pv[j];
                rq += q;
                cols[j] += pv[j];
                colq[j] += q;
            }
            rs = __reduce_add_sync(0xffffffffu, rs);      // row sums of the tile (< 2^32: 128 * 255^2)
            rq = __reduce_add_sync(0xffffffffu, rq);
            if (lane == 0) {
                rowsum[r] = rs;
                rowsum[BAND + r] = rq;
            }
        }
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        red_s[warp][4 * lane + j] = cols[j];
        red_q[warp][4 * lane + j] = colq[j];
    }
    __syncthreads();
    if (threadIdx.x < CHUNK) {
        const int xx = x0 + threadIdx.x;
        if (xx < L.W) {
            uint32_t ts = 0, tq = 0;
#pragma unroll
            for (int w = 0; w < 8; ++w) {
                ts += red_s[w][threadIdx.x];
                tq += red_q[w][threadIdx.x];
            }
            uint32_t* col = s.col + (size_t)g * p.col_frame + L.col_off + (size_t)b * 2 * L.W;
            col[xx] = ts;
            col[L.W + xx] = tq;
        }
    }
}

// ---------------------------------------------------------------- K1s: exclusive carries
// blockIdx.y <  n_levels: column carries of level y (exclusive over bands)
// blockIdx.y >= n_levels: row carries of level y - n_levels (exclusive over chunks)
__global__ void __launch_bounds__(K1_THREADS) k_carry(const __grid_constant__ PlanDev p, K1Scratch s) {
    const int g = blockIdx.z;
    const int i = blockIdx.x * K1_THREADS + threadIdx.x;
    // exclusive scan of n strided pairs (plane 0 at v[0], plane 1 at v[off]); loads are batched
    // 16 at a time so the latency is paid once per batch, not once per element
    auto scan_pairs = [](uint32_t* v, int n, size_t stride, size_t off) {
        uint32_t rs = 0, rq = 0;
        for (int b0 = 0; b0 < n; b0 += 16) {
            uint32_t a[16], q[16];
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                if (b0 + j < n) {
                    a[j] = v[(size_t)(b0 + j) * stride];
                    q[j] = v[(size_t)(b0 + j) * stride + off];
                }
            }
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                if (b0 + j < n) {
                    v[(size_t)(b0 + j) * stride] = rs;
                    v[(size_t)(b0 + j) * stride + off] = rq;
                    rs += a[j];
                    rq += q[j];
                }
            }
        }
    };
    if ((int)blockIdx.y < p.n_levels) {
        const LevelDev& L = p.lv[blockIdx.y];
        if (i >= L.W) return;
        scan_pairs(s.col + (size_t)g * p.col_frame + L.col_off + i, L.nbands, (size_t)2 * L.W, (size_t)L.W);
    } else {
        const LevelDev& L = p.lv[blockIdx.y - p.n_levels];
        const int b = i / BAND, r = i % BAND;
        if (b >= L.nbands) return;
        scan_pairs(s.row + (size_t)g * p.row_frame + L.row_off + (size_t)b * L.nchunks * 2 * BAND + r, L.nchunks,
                   (size_t)2 * BAND, (size_t)BAND);
    }
}

// ---------------------------------------------------------------- K1c: tile corners
// corner[band][chunk][plane] = ii at (y0, x0) = sum_{x < x0} colcarry_band[x]  (u64: exact for
// the canonical u64 sqii; the internal workspace keeps its low 32 bits)
__global__ void __launch_bounds__(K1_THREADS) k_corner(const __grid_constant__ PlanDev p, K1Scratch s) {
    const int g = blockIdx.y;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gb = blockIdx.x * (K1_THREADS / 32) + warp;      // band index within the frame
    if (gb >= p.bands_per_frame) return;
    int k = 0;
    while (k + 1 < p.n_levels && p.lv[k + 1].band0 <= gb) ++k;
    const LevelDev& L = p.lv[k];
    const int b = gb - L.band0;
    const uint32_t* col = s.col + (size_t)g * p.col_frame + L.col_off + (size_t)b * 2 * L.W;
    unsigned long long* cor = s.cor + (size_t)g * p.cor_frame + L.cor_off + (size_t)b * L.nchunks * 2;
    unsigned long long run_s = 0, run_q = 0;
    for (int c = 0; c < L.nchunks; ++c) {
        unsigned long long ts = 0, tq = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int x = c * CHUNK + 4 * lane + j;
            if (x < L.W) {
                ts += col[x];
                tq += col[L.W + x];
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            ts += __shfl_xor_sync(0xffffffffu, ts, o);
            tq += __shfl_xor_sync(0xffffffffu, tq, o);
        }
        if (lane == 0) {
            cor[2 * c] = run_s;
            cor[2 * c + 1] = run_q;
        }
        run_s += ts;
        run_q += tq;
    }
}

// ---------------------------------------------------------------- K1b: tile integral
// CANON = false: internal layout (u32 ii + u32 sqii mod 2^32 in the group workspace planes)
// CANON = true : fd_integral output (u32 ii, u64 sqii, caller pitch)
template <bool CANON>
struct BandOut;
template <>
struct BandOut<false> {
    using QT = uint32_t;
};
template <>
struct BandOut<true> {
    using QT = unsigned long long;
};

// Row phase: thread (r, sg) owns row r of the band and the 16 columns x0 + 16 sg .. of the chunk
// (one 16-B load of the level image, pitch PB): exclusive prefixes of p and p^2 in registers, the
// 8 segments of a row exchange exclusive offsets with 3 shuffles, plus the row carry (pixels left
// of the chunk).  Column phase: thread per (column, plane) walks down the band adding the row
// prefixes to the tile's top row ii[y0][X] and stores each ii / sqii entry once (a warp stores
// 32 consecutive entries of a row: 128 or 256 B).
template <bool CANON>
__global__ void __launch_bounds__(K1_THREADS) k_tile(const uint8_t* __restrict__ frames, const __grid_constant__ PlanDev p,
                                                     K1Scratch s, uint32_t* __restrict__ ws,
                                                     uint32_t* __restrict__ out_ii,
                                                     unsigned long long* __restrict__ out_sq, int out_pitch) {
    using QT = typename BandOut<CANON>::QT;
    static_assert(K1_THREADS == 8 * BAND && CHUNK == 8 * 16, "row phase: 8 segments of 16 columns per row");
    __shared__ __align__(16) uint32_t rp_s[BAND][CHUNK];
    __shared__ __align__(16) uint32_t rp_q[BAND][CHUNK];   // row prefixes of p^2: < W * 255^2 < 2^32, exact
    __shared__ __align__(16) uint32_t top_s[CHUNK];
    __shared__ __align__(16) QT top_q[CHUNK];
    (void)frames;
    const int g = blockIdx.y;
    const int k = find_level_k1(p, blockIdx.x);
    const LevelDev& L = p.lv[k];
    const int tl = blockIdx.x - L.k1t0;
    const int b = tl / L.nchunks, c = tl % L.nchunks;
    const int y0 = b * BAND, rows = min(BAND, L.H - y0);
    const int x0 = c * CHUNK;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const uint32_t* carry = s.col + (size_t)g * p.col_frame + L.col_off + (size_t)b * 2 * L.W;
    const uint32_t* rowc = s.row + (size_t)g * p.row_frame + L.row_off + (size_t)(b * L.nchunks + c) * 2 * BAND;
    const unsigned long long* cor = s.cor + (size_t)g * p.cor_frame + L.cor_off + (size_t)(b * L.nchunks + c) * 2;
    const uint8_t* lvl = s.lvl + (size_t)g * p.lvl_frame + L.lvl_off;

    // ---- row phase
    {
        const int r = tid >> 3, sg = tid & 7;
        const int xs = x0 + 16 * sg;
        uint4 w = make_uint4(0u, 0u, 0u, 0u);
        if (r < rows && xs < L.PB) w = __ldg(reinterpret_cast<const uint4*>(lvl + (size_t)(y0 + r) * L.PB + xs));
        const uint32_t wd[4] = {w.x, w.y, w.z, w.w};
        uint32_t ps[16], pq[16];
        uint32_t ts = 0, tq = 0;
#pragma unroll
        for (int i = 0; i < 16; ++i) {      // exclusive: ii column X sums the pixels x < X
            const uint32_t v = (wd[i >> 2] >> (8 * (i & 3))) & 255u;
            ps[i] = ts;
            pq[i] = tq;
            ts += v;
            tq += v * v;
        }
        uint32_t is = ts, iq = tq;
#pragma unroll
        for (int d = 1; d < 8; d <<= 1) {
            const uint32_t a = __shfl_up_sync(0xffffffffu, is, d, 8);
            const uint32_t q = __shfl_up_sync(0xffffffffu, iq, d, 8);
            if (sg >= d) {
                is += a;
                iq += q;
            }
        }
        const uint32_t bs = (r < rows ? rowc[r] : 0u) + is - ts;
        const uint32_t bq = (r < rows ? rowc[BAND + r] : 0u) + iq - tq;
#pragma unroll
        for (int i = 0; i < 16; i += 4) {
            *reinterpret_cast<uint4*>(&rp_s[r][16 * sg + i]) =
                make_uint4(bs + ps[i], bs + ps[i + 1], bs + ps[i + 2], bs + ps[i + 3]);
            *reinterpret_cast<uint4*>(&rp_q[r][16 * sg + i]) =
                make_uint4(bq + pq[i], bq + pq[i + 1], bq + pq[i + 2], bq + pq[i + 3]);
        }
    }
    if (warp == 0) {     // top row ii[y0][X] = corner + sum_{x0 <= x < X} carry[x]
        const int x = x0 + 4 * lane;
        uint32_t cv[4];
        QT cq[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            cv[j] = x + j < L.W ? carry[x + j] : 0u;
            cq[j] = x + j < L.W ? (QT)carry[L.W + x + j] : (QT)0;
        }
        uint32_t es[4], ts = 0;
        QT eq[4], tq = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            es[j] = ts;
            eq[j] = tq;
            ts += cv[j];
            tq += cq[j];
        }
        uint32_t is = ts;
        QT iq = tq;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t a = __shfl_up_sync(0xffffffffu, is, d);
            const QT q = __shfl_up_sync(0xffffffffu, iq, d);
            if (lane >= d) {
                is += a;
                iq += q;
            }
        }
        const uint32_t bs = (uint32_t)cor[0] + is - ts;
        const QT bq = (QT)cor[1] + iq - tq;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            top_s[4 * lane + j] = bs + es[j];
            top_q[4 * lane + j] = bq + eq[j];
        }
    }
    __syncthreads();

    // ---- column phase: thread (plane, column)
    const int col = tid & (CHUNK - 1), plane = tid / CHUNK;
    const int X = x0 + col;
    const int P = CANON ? out_pitch : L.P;
    if (X >= P) return;
    if (plane == 0) {
        uint32_t* o = CANON ? out_ii + (size_t)g * (L.H + 1) * out_pitch
                            : ws + L.ws_off + (size_t)g * 2 * (size_t)(L.H + 1) * L.P;
        if (b == 0) o[X] = 0u;                    // ii row 0
        uint32_t acc = top_s[col];
        o += (size_t)(y0 + 1) * P + X;
#pragma unroll 8
        for (int r = 0; r < rows; ++r) {
            acc += rp_s[r][col];
            o[(size_t)r * P] = acc;
        }
    } else {
        QT* o;
        if constexpr (CANON)
            o = reinterpret_cast<QT*>(out_sq) + (size_t)g * (L.H + 1) * out_pitch;
        else
            o = reinterpret_cast<QT*>(ws + L.ws_off + (size_t)g * 2 * (size_t)(L.H + 1) * L.P + (size_t)(L.H + 1) * L.P);
        if (b == 0) o[X] = (QT)0;
        QT acc = top_q[col];
        o += (size_t)(y0 + 1) * P + X;
#pragma unroll 8
        for (int r = 0; r < rows; ++r) {
            acc += (QT)rp_q[r][col];
            o[(size_t)r * P] = acc;
        }
    }
}

// ---------------------------------------------------------------- f1: level images
// The group workspace of the f1 path holds only the level images: u8, level-major
// out + L.u8_off + (g * H_k + y) * PB_k + x, each row zero-padded to PB_k (a 16-B multiple, for
// the TMA boxes of k_f1).  Pixels are resampled from the frame (R2) and, when the cascade asks for
// it, filtered (R3b) with exactly the arithmetic k_marg uses for K1.  One CTA per (frame, K1
// tile of 32 rows x 128 columns); a lane writes 4 pixels as one aligned word.
__global__ void __launch_bounds__(K1_THREADS) k_level(const uint8_t* __restrict__ frames, const __grid_constant__ PlanDev p,
                                                      uint8_t* __restrict__ out) {
    __shared__ uint8_t raw[BAND + 2][CHUNK + 4];       // filtering stage: resampled rows with a 1-px halo
    __shared__ __align__(16) uint8_t src[SRC_ROWS * SRC_PITCH];   // staged source region
    const int g = blockIdx.y;
    const int k = find_level_k1(p, blockIdx.x);
    const LevelDev& L = p.lv[k];
    const int tl = blockIdx.x - L.k1t0;
    const int b = tl / L.nchunks, c = tl % L.nchunks;
    const int y0 = b * BAND, rows = min(BAND, L.H - y0);
    const int x0 = c * CHUNK;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint8_t* frame = frames + (size_t)g * p.H * p.pitch;
    const int x = x0 + 4 * lane;
    const bool staged = !p.filter && p.aligned16 && L.r16 != 65536 && L.r16 <= STAGE_R16_MAX;
    ColSample cs[4];
    int so[4], sax[4];
    SrcStage sst{0, 0};
    if (staged) {
        sst = stage_source(frame, p, L, y0, rows, x0, src);
#pragma unroll
        for (int j = 0; j < 4; ++j) so[j] = src_coord(min(x + j, L.W - 1), L.r16, p.W, &sax[j]) - sst.xa;
    } else if (L.r16 != 65536) {
#pragma unroll
        for (int j = 0; j < 4; ++j) cs[j] = col_sample(p.W, L.r16, min(x + j, L.W - 1));
    }
    uint8_t* o = out + L.u8_off + ((size_t)g * L.H + y0) * L.PB;
    if (p.filter) {
        for (int r = warp; r < rows + 2; r += K1_THREADS / 32) {
            const int yy = min(max(y0 - 1 + r, 0), L.H - 1);
            for (int q = lane; q < CHUNK + 2; q += 32) {
                const int xx = min(max(x0 - 1 + q, 0), L.W - 1);
                raw[r][q] = (uint8_t)level_pixel(frame, p.pitch, p.W, p.H, L.r16, xx, yy);
            }
        }
        __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < BAND / 8; ++i) {
        const int r = warp + 8 * i;
        if (r < rows && x < L.PB) {
            uint32_t pv[4];
            if (p.filter) {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int q = x + j - x0 + 1;
                    uint32_t v = 0;
                    if (x + j < L.W) {
#pragma unroll
                        for (int dy = 0; dy < 3; ++dy) {
                            const uint32_t h = raw[r + dy][q - 1] + 2u * raw[r + dy][q] + raw[r + dy][q + 1];
                            v += (dy == 1 ? 2u : 1u) * h;
                        }
                        v = (v + 8u) >> 4;
                    }
                    pv[j] = v;
                }
            } else if (staged) {
                staged_row_pixels(src, p, L, sst, y0 + r, x, so, sax, pv);
            } else {
                tile_row_pixels(frame, p, L, y0 + r, x, cs, pv);
            }
            *reinterpret_cast<uint32_t*>(o + (size_t)r * L.PB + x) = pv[0] | (pv[1] << 8) | (pv[2] << 16) | (pv[3] << 24);
        }
    }
}

// ---------------------------------------------------------------- fd_build_pyramid
__global__ void __launch_bounds__(256) k_pyramid(const uint8_t* __restrict__ frames, const __grid_constant__ PlanDev p,
                                                 uint8_t* __restrict__ out, long long frame_stride) {
    const int k = blockIdx.y, g = blockIdx.z;
    const LevelDev& L = p.lv[k];
    const long long npx = (long long)L.W * L.H;
    const uint8_t* frame = frames + (size_t)g * p.H * p.pitch;
    uint8_t* o = out + (size_t)g * frame_stride + L.col_off;    // col_off reused as the level byte offset
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < npx; i += (long long)gridDim.x * blockDim.x) {
        const int y = (int)(i / L.W), x = (int)(i % L.W);
        o[i] = (uint8_t)level_pixel(frame, p.pitch, p.W, p.H, L.r16, x, y);
    }
}

// ---------------------------------------------------------------- launchers
cudaError_t launch_k1_marg(const uint8_t* frames, const PlanDev& plan, int g_frames, const K1Scratch& s, cudaStream_t st) {
    dim3 grid(plan.k1tiles_per_frame, g_frames);
    k_marg<<<grid, K1_THREADS, 0, st>>>(frames, plan, s);
    return cudaGetLastError();
}

cudaError_t launch_k1_carry(const PlanDev& plan, int g_frames, const K1Scratch& s, cudaStream_t st) {
    int maxb = 0;
    for (int k = 0; k < plan.n_levels; ++k) maxb = plan.lv[k].nbands > maxb ? plan.lv[k].nbands : maxb;
    const int span = plan.maxW > maxb * BAND ? plan.maxW : maxb * BAND;
    dim3 grid((span + K1_THREADS - 1) / K1_THREADS, 2 * plan.n_levels, g_frames);
    k_carry<<<grid, K1_THREADS, 0, st>>>(plan, s);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    dim3 g2((plan.bands_per_frame + K1_THREADS / 32 - 1) / (K1_THREADS / 32), g_frames);
    k_corner<<<g2, K1_THREADS, 0, st>>>(plan, s);
    return cudaGetLastError();
}

cudaError_t launch_k1_tiles(const uint8_t* frames, const PlanDev& plan, int g_frames, const K1Scratch& s, uint32_t* ws,
                            cudaStream_t st) {
    dim3 grid(plan.k1tiles_per_frame, g_frames);
    k_tile<false><<<grid, K1_THREADS, 0, st>>>(frames, plan, s, ws, nullptr, nullptr, 0);
    return cudaGetLastError();
}

cudaError_t launch_k1_tiles_canonical(const uint8_t* img, const PlanDev& plan, int n, const K1Scratch& s, uint32_t* ii,
                                      uint64_t* sqii, int out_pitch, cudaStream_t st) {
    dim3 grid(plan.k1tiles_per_frame, n);
    k_tile<true><<<grid, K1_THREADS, 0, st>>>(img, plan, s, nullptr, ii, reinterpret_cast<unsigned long long*>(sqii),
                                              out_pitch);
    return cudaGetLastError();
}

cudaError_t launch_levels(const uint8_t* frames, const PlanDev& plan, int g_frames, uint8_t* out, cudaStream_t st) {
    dim3 grid(plan.k1tiles_per_frame, g_frames);
    k_level<<<grid, K1_THREADS, 0, st>>>(frames, plan, out);
    return cudaGetLastError();
}

cudaError_t launch_pyramid(const uint8_t* frames, const PlanDev& plan, int n, uint8_t* levels, long long frame_stride,
                           const long long*, cudaStream_t st) {
    dim3 grid(64, plan.n_levels, n);
    k_pyramid<<<grid, 256, 0, st>>>(frames, plan, levels, frame_stride);
    return cudaGetLastError();
}

}  // namespace fdk
