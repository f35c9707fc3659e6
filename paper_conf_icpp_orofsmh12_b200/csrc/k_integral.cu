// k_integral.cu -- K1: pyramid scaling fused with integral + squared-integral images.
//
// Paper: "the scaling stage generates n resized images by subsampling the decompressed
// frame ... tex2D linear interpolation"; "integral images are computed ... with a
// combination of parallel prefix sum [17][18] and matrix transposition operations [19]"
// (P:L368-384).  B200 design: no level image and no transpose
// is materialised.  Each level is cut into 32-row bands; a band CTA resamples its pixels
// straight from the frame (exact integer bilinear, reading R2), does warp-shuffle row scans,
// stages the row prefixes in shared memory and runs a coalesced, vectorised (uint4) column
// scan that adds the carry of all rows above.  The carry comes from two light kernels
// (per-band column sums, then an exclusive scan over bands), so ii/sqii are written to HBM
// exactly once.
#include <cub/cub.cuh>

#include "fd_internal.h"

namespace fdk {

// ---------------------------------------------------------------- scaling (reading R2)
struct RowSample {
    const uint8_t* r0;
    const uint8_t* r1;
    int ay;
};

__device__ __forceinline__ RowSample row_sample(const uint8_t* frame, int pitch, int H, int r16, int y) {
    const long long sy = ((2LL * y + 1) * (long long)r16 - 65536) >> 1;
    int y0 = (int)(sy >> 16);
    y0 = y0 < H - 1 ? y0 : H - 1;
    const int y1 = y0 + 1 < H ? y0 + 1 : H - 1;
    RowSample s;
    s.r0 = frame + (size_t)y0 * pitch;
    s.r1 = frame + (size_t)y1 * pitch;
    s.ay = (int)((sy >> 8) & 255);
    return s;
}

struct ColSample {
    int x0, x1, ax;
};

__device__ __forceinline__ ColSample col_sample(int W, int r16, int x) {
    const long long sx = ((2LL * x + 1) * (long long)r16 - 65536) >> 1;
    int x0 = (int)(sx >> 16);
    x0 = x0 < W - 1 ? x0 : W - 1;
    ColSample c;
    c.x0 = x0;
    c.x1 = x0 + 1 < W ? x0 + 1 : W - 1;
    c.ax = (int)((sx >> 8) & 255);
    return c;
}

// p = (p00(256-ax)(256-ay) + p01 ax(256-ay) + p10(256-ax)ay + p11 ax ay + 2^15) >> 16,
// evaluated as two horizontal lerps then one vertical (identical in exact integer arithmetic).
__device__ __forceinline__ uint32_t bilinear(const RowSample& r, const ColSample& c) {
    const int p00 = __ldg(r.r0 + c.x0), p01 = __ldg(r.r0 + c.x1);
    const int p10 = __ldg(r.r1 + c.x0), p11 = __ldg(r.r1 + c.x1);
    const int h0 = p00 * (256 - c.ax) + p01 * c.ax;
    const int h1 = p10 * (256 - c.ax) + p11 * c.ax;
    return (uint32_t)((h0 * (256 - r.ay) + h1 * r.ay + 32768) >> 16);
}

__device__ __forceinline__ uint32_t level_pixel(const uint8_t* frame, int pitch, int srcW, int srcH, int r16,
                                                int x, int y) {
    if (r16 == 65536) return __ldg(frame + (size_t)y * pitch + x);   // level 0: identity
    const RowSample r = row_sample(frame, pitch, srcH, r16, y);
    return bilinear(r, col_sample(srcW, r16, x));
}

__device__ __forceinline__ int find_level_band(const PlanDev& p, int b) {
    int k = 0;
    while (k + 1 < p.n_levels && p.lv[k + 1].band0 <= b) ++k;
    return k;
}

// ---------------------------------------------------------------- K1a: per-band column sums
__global__ void __launch_bounds__(K1_THREADS) k_colsum(const uint8_t* __restrict__ frames,
                                                       const __grid_constant__ PlanDev p,
                                                       uint32_t* __restrict__ colbuf) {
    const int g = blockIdx.y;
    const int k = find_level_band(p, blockIdx.x);
    const LevelDev& L = p.lv[k];
    const int b = blockIdx.x - L.band0;
    const int y0 = b * BAND, rows = min(BAND, L.H - y0);
    const uint8_t* frame = frames + (size_t)g * p.H * p.pitch;
    uint32_t* col = colbuf + (size_t)g * p.col_frame + L.col_off + (size_t)b * 2 * L.W;
    for (int x = threadIdx.x; x < L.W; x += K1_THREADS) {
        uint32_t s = 0, q = 0;
        if (L.r16 == 65536) {
            for (int r = 0; r < rows; ++r) {
                const uint32_t v = __ldg(frame + (size_t)(y0 + r) * p.pitch + x);
                s += v;
                q += v * v;
            }
        } else {
            const ColSample c = col_sample(p.W, L.r16, x);
            for (int r = 0; r < rows; ++r) {
                const uint32_t v = bilinear(row_sample(frame, p.pitch, p.H, L.r16, y0 + r), c);
                s += v;
                q += v * v;
            }
        }
        col[x] = s;
        col[L.W + x] = q;
    }
}

// ---------------------------------------------------------------- K1s: exclusive carry over bands
__global__ void __launch_bounds__(K1_THREADS) k_carry(const __grid_constant__ PlanDev p, uint32_t* __restrict__ colbuf) {
    const int k = blockIdx.y, g = blockIdx.z;
    const LevelDev& L = p.lv[k];
    const int x = blockIdx.x * K1_THREADS + threadIdx.x;
    if (x >= L.W) return;
    uint32_t* col = colbuf + (size_t)g * p.col_frame + L.col_off + x;
    uint32_t cs = 0, cq = 0;
    for (int b = 0; b < L.nbands; ++b) {
        uint32_t* c = col + (size_t)b * 2 * L.W;
        const uint32_t s = c[0], q = c[L.W];
        c[0] = cs;
        c[L.W] = cq;
        cs += s;
        cq += q;
    }
}

// ---------------------------------------------------------------- K1b: band integral
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

template <bool CANON>
__global__ void __launch_bounds__(K1_THREADS) k_band(const uint8_t* __restrict__ frames, const __grid_constant__ PlanDev p,
                                                     const uint32_t* __restrict__ colbuf, uint32_t* __restrict__ ws,
                                                     uint32_t* __restrict__ out_ii,
                                                     unsigned long long* __restrict__ out_sq, int out_pitch) {
    using QT = typename BandOut<CANON>::QT;
    __shared__ __align__(16) uint32_t rp_s[BAND][CHUNK];
    __shared__ __align__(16) uint32_t rp_q[BAND][CHUNK];
    __shared__ __align__(16) uint32_t seg_s[8][CHUNK];
    __shared__ __align__(16) QT seg_q[8][CHUNK];
    __shared__ __align__(16) uint32_t top_s[CHUNK];
    __shared__ __align__(16) QT top_q[CHUNK];

    const int g = blockIdx.y;
    const int k = find_level_band(p, blockIdx.x);
    const LevelDev& L = p.lv[k];
    const int b = blockIdx.x - L.band0;
    const int y0 = b * BAND, rows = min(BAND, L.H - y0);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint8_t* frame = frames + (size_t)g * p.H * p.pitch;
    const uint32_t* carry = colbuf + (size_t)g * p.col_frame + L.col_off + (size_t)b * 2 * L.W;

    // output addressing
    const int P = CANON ? out_pitch : L.P;
    uint32_t* o_ii;
    QT* o_sq;
    if constexpr (CANON) {
        o_ii = out_ii + (size_t)g * (L.H + 1) * out_pitch;
        o_sq = reinterpret_cast<QT*>(out_sq + (size_t)g * (L.H + 1) * out_pitch);
    } else {
        const size_t plane = (size_t)(L.H + 1) * L.P;
        o_ii = ws + L.ws_off + (size_t)g * 2 * plane;
        o_sq = reinterpret_cast<QT*>(o_ii + plane);
    }

    uint32_t rc_s[4] = {0, 0, 0, 0}, rc_q[4] = {0, 0, 0, 0};   // row carries (pixels < x0)
    uint32_t tc_s = 0;                                          // top-row carry (warp 0)
    QT tc_q = 0;

    const int q4 = threadIdx.x & 31;        // column-phase: column group (4 ii columns)
    const int sg = threadIdx.x >> 5;        // column-phase: 4-row segment

    for (int x0 = 0; x0 < P; x0 += CHUNK) {
        // ---- row phase: warp-shuffle scans of 4 rows per warp (+ the carry row for warp 0)
        ColSample cs[4];
        if (L.r16 != 65536) {
#pragma unroll
            for (int j = 0; j < 4; ++j) cs[j] = col_sample(p.W, L.r16, min(x0 + 4 * lane + j, L.W - 1));
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int r = warp + 8 * i;
            if (r < rows) {
                const int y = y0 + r;
                uint32_t pv[4];
                if (L.r16 == 65536) {
                    const uint8_t* row = frame + (size_t)y * p.pitch;
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int x = x0 + 4 * lane + j;
                        pv[j] = x < L.W ? __ldg(row + x) : 0u;
                    }
                } else {
                    const RowSample rs = row_sample(frame, p.pitch, p.H, L.r16, y);
#pragma unroll
                    for (int j = 0; j < 4; ++j) pv[j] = (x0 + 4 * lane + j < L.W) ? bilinear(rs, cs[j]) : 0u;
                }
                uint32_t es[4], eq[4], ts = 0, tq = 0;
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    es[j] = ts;
                    eq[j] = tq;
                    ts += pv[j];
                    tq += pv[j] * pv[j];
                }
                uint32_t is = ts, iq = tq;    // warp inclusive scan of lane totals
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const uint32_t a = __shfl_up_sync(0xffffffffu, is, d);
                    const uint32_t c = __shfl_up_sync(0xffffffffu, iq, d);
                    if (lane >= d) {
                        is += a;
                        iq += c;
                    }
                }
                const uint32_t bs = rc_s[i] + is - ts, bq = rc_q[i] + iq - tq;
                *reinterpret_cast<uint4*>(&rp_s[r][4 * lane]) = make_uint4(bs + es[0], bs + es[1], bs + es[2], bs + es[3]);
                *reinterpret_cast<uint4*>(&rp_q[r][4 * lane]) = make_uint4(bq + eq[0], bq + eq[1], bq + eq[2], bq + eq[3]);
                rc_s[i] += __shfl_sync(0xffffffffu, is, 31);
                rc_q[i] += __shfl_sync(0xffffffffu, iq, 31);
            }
        }
        if (warp == 0) {     // top row ii[y0][X] = sum_{x<X} carry[x]
            uint32_t cv[4];
            QT cq[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int x = x0 + 4 * lane + j;
                cv[j] = x < L.W ? carry[x] : 0u;
                cq[j] = x < L.W ? (QT)carry[L.W + x] : (QT)0;
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
                const QT c = __shfl_up_sync(0xffffffffu, iq, d);
                if (lane >= d) {
                    is += a;
                    iq += c;
                }
            }
            const uint32_t bs = tc_s + is - ts;
            const QT bq = tc_q + iq - tq;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                top_s[4 * lane + j] = bs + es[j];
                top_q[4 * lane + j] = bq + eq[j];
            }
            tc_s += __shfl_sync(0xffffffffu, is, 31);
            tc_q += __shfl_sync(0xffffffffu, iq, 31);
        }
        __syncthreads();

        // ---- column phase: thread (q4, sg) owns ii columns x0+4q4.. and rows 4sg..4sg+3
        {
            uint32_t ss[4] = {0, 0, 0, 0};
            QT sq[4] = {0, 0, 0, 0};
#pragma unroll
            for (int rr = 0; rr < 4; ++rr) {
                const int r = 4 * sg + rr;
                if (r < rows) {
                    const uint4 a = *reinterpret_cast<const uint4*>(&rp_s[r][4 * q4]);
                    const uint4 c = *reinterpret_cast<const uint4*>(&rp_q[r][4 * q4]);
                    ss[0] += a.x; ss[1] += a.y; ss[2] += a.z; ss[3] += a.w;
                    sq[0] += c.x; sq[1] += c.y; sq[2] += c.z; sq[3] += c.w;
                }
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                seg_s[sg][4 * q4 + j] = ss[j];
                seg_q[sg][4 * q4 + j] = sq[j];
            }
        }
        __syncthreads();
        {
            uint32_t os[4];
            QT oq[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                os[j] = top_s[4 * q4 + j];
                oq[j] = top_q[4 * q4 + j];
            }
            for (int s2 = 0; s2 < sg; ++s2) {
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    os[j] += seg_s[s2][4 * q4 + j];
                    oq[j] += seg_q[s2][4 * q4 + j];
                }
            }
            const int X = x0 + 4 * q4;
            if (b == 0 && sg == 0 && X < P) {       // ii row 0 is zero
                *reinterpret_cast<uint4*>(o_ii + X) = make_uint4(0, 0, 0, 0);
                if constexpr (CANON) {
                    *reinterpret_cast<ulonglong2*>(o_sq + X) = make_ulonglong2(0, 0);
                    *reinterpret_cast<ulonglong2*>(o_sq + X + 2) = make_ulonglong2(0, 0);
                } else {
                    *reinterpret_cast<uint4*>(o_sq + X) = make_uint4(0, 0, 0, 0);
                }
            }
#pragma unroll
            for (int rr = 0; rr < 4; ++rr) {
                const int r = 4 * sg + rr;
                if (r < rows) {
                    const uint4 a = *reinterpret_cast<const uint4*>(&rp_s[r][4 * q4]);
                    const uint4 c = *reinterpret_cast<const uint4*>(&rp_q[r][4 * q4]);
                    os[0] += a.x; os[1] += a.y; os[2] += a.z; os[3] += a.w;
                    oq[0] += c.x; oq[1] += c.y; oq[2] += c.z; oq[3] += c.w;
                    if (X < P) {
                        const size_t o = (size_t)(y0 + r + 1) * P + X;
                        *reinterpret_cast<uint4*>(o_ii + o) = make_uint4(os[0], os[1], os[2], os[3]);
                        if constexpr (CANON) {
                            *reinterpret_cast<ulonglong2*>(o_sq + o) = make_ulonglong2(oq[0], oq[1]);
                            *reinterpret_cast<ulonglong2*>(o_sq + o + 2) = make_ulonglong2(oq[2], oq[3]);
                        } else {
                            *reinterpret_cast<uint4*>(o_sq + o) = make_uint4(oq[0], oq[1], oq[2], oq[3]);
                        }
                    }
                }
            }
        }
        __syncthreads();
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
cudaError_t launch_colsum(const uint8_t* frames, const PlanDev& plan, int g_frames, uint32_t* colbuf, cudaStream_t st) {
    dim3 grid(plan.bands_per_frame, g_frames);
    k_colsum<<<grid, K1_THREADS, 0, st>>>(frames, plan, colbuf);
    return cudaGetLastError();
}

cudaError_t launch_carry(const PlanDev& plan, int g_frames, uint32_t* colbuf, cudaStream_t st) {
    dim3 grid((plan.maxW + K1_THREADS - 1) / K1_THREADS, plan.n_levels, g_frames);
    k_carry<<<grid, K1_THREADS, 0, st>>>(plan, colbuf);
    return cudaGetLastError();
}

cudaError_t launch_band(const uint8_t* frames, const PlanDev& plan, int g_frames, const uint32_t* colbuf, uint32_t* ws,
                        cudaStream_t st) {
    dim3 grid(plan.bands_per_frame, g_frames);
    k_band<false><<<grid, K1_THREADS, 0, st>>>(frames, plan, colbuf, ws, nullptr, nullptr, 0);
    return cudaGetLastError();
}

cudaError_t launch_integral_canonical(const uint8_t* img, const PlanDev& plan, int n, const uint32_t* colbuf,
                                      uint32_t* ii, uint64_t* sqii, int out_pitch, cudaStream_t st) {
    dim3 grid(plan.bands_per_frame, n);
    k_band<true><<<grid, K1_THREADS, 0, st>>>(img, plan, colbuf, nullptr, ii,
                                               reinterpret_cast<unsigned long long*>(sqii), out_pitch);
    return cudaGetLastError();
}

cudaError_t launch_pyramid(const uint8_t* frames, const PlanDev& plan, int n, uint8_t* levels, long long frame_stride,
                           const long long*, cudaStream_t st) {
    dim3 grid(64, plan.n_levels, n);
    k_pyramid<<<grid, 256, 0, st>>>(frames, plan, levels, frame_stride);
    return cudaGetLastError();
}

}  // namespace fdk
