// k_common.cuh -- device helpers shared by the K2 cascade kernels (k_cascade.cu, k_cascade_ws.cu):
// mbarrier / TMA wrappers, stump-record accessors and the exact stump / stage evaluators
// (oracle c7/c8: (float)f < theta*nf ? left : right, fp32 stage sums in stump order, no FMA).
#pragma once
#include "fd_internal.h"

namespace fdk {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* map, int x, int y, int z, int w, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(
            smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(z), "r"(w), "r"(smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ int corner_word(const uint4& a, const uint4& b, const uint4& c, int i) {
    const uint4& v = i < 4 ? a : (i < 8 ? b : c);
    const int j = i & 3;
    return (int)(j == 0 ? v.x : (j == 1 ? v.y : (j == 2 ? v.z : v.w)));
}

// Record accessors: word4 i of the packed stump records (4 x uint4 per stump).
struct GlobalRec {                 // global memory, read-only path (lane-varying indices)
    const uint4* s;
    __device__ __forceinline__ uint4 operator()(int i) const { return __ldg(s + i); }
};
struct ParamRec {                  // kernel-parameter constant bank (warp-uniform indices)
    const CascadeParams& p;
    __device__ __forceinline__ uint4 operator()(int i) const { return p.prec[i]; }
};

// One stump for one window with a compile-time corner count MC >= the stump's corners: the
// unused corner words are zero (offset 0, coefficient 0), so the loop is branch-free.
template <int MC, class R>
__device__ __forceinline__ float eval_stump_mc(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int j) {
    const uint4 h = rec(4 * j);
    const uint4 c0 = rec(4 * j + 1);
    const uint4 c1 = MC > 4 ? rec(4 * j + 2) : make_uint4(0, 0, 0, 0);
    const uint4 c2 = MC > 8 ? rec(4 * j + 3) : make_uint4(0, 0, 0, 0);
    uint32_t f = 0;
#pragma unroll
    for (int c = 0; c < MC; ++c) {
        const int w = corner_word(c0, c1, c2, c);
        f += (uint32_t)(w >> 16) * *reinterpret_cast<const uint32_t*>(reinterpret_cast<const char*>(T + b) + (w & 0xffff));
    }
    const float t = __fmul_rn(__int_as_float((int)h.y), nf);
    return (__int2float_rn((int)f) < t) ? __int_as_float((int)h.z) : __int_as_float((int)h.w);
}

// One stage for one window: sum_j leaf_j in stump order (oracle c7/c8).  Stumps are
// independent until the ordered fp32 additions, so four are evaluated per iteration.
template <int MC, class R>
__device__ __forceinline__ float eval_stage_mc(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int first,
                                               int n) {
    float sum = 0.0f;
    int j = 0;
    for (; j + 4 <= n; j += 4) {
        const float l0 = eval_stump_mc<MC>(T, b, nf, rec, first + j);
        const float l1 = eval_stump_mc<MC>(T, b, nf, rec, first + j + 1);
        const float l2 = eval_stump_mc<MC>(T, b, nf, rec, first + j + 2);
        const float l3 = eval_stump_mc<MC>(T, b, nf, rec, first + j + 3);
        sum = __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(sum, l0), l1), l2), l3);
    }
    for (; j < n; ++j) sum = __fadd_rn(sum, eval_stump_mc<MC>(T, b, nf, rec, first + j));
    return sum;
}

// mc = the stage's largest corner count (StageDev::mc); dispatch to a padded, unrolled body
template <class R>
__device__ __forceinline__ float eval_stage(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int first, int n,
                                            int mc) {
    if (mc <= 4) return eval_stage_mc<4>(T, b, nf, rec, first, n);
    if (mc <= 6) return eval_stage_mc<6>(T, b, nf, rec, first, n);
    if (mc <= 8) return eval_stage_mc<8>(T, b, nf, rec, first, n);
    if (mc <= 9) return eval_stage_mc<9>(T, b, nf, rec, first, n);
    return eval_stage_mc<MAX_CORNERS>(T, b, nf, rec, first, n);
}

// One stage for one window evaluated by a group of GL = 2^lg lanes (lane-aligned within a warp).
// Per chunk of GL*LC stumps, lane q of the group evaluates stumps c0 + q + GL*r (r < LC,
// independent, so LC loads are in flight) and parks the leaves at lv[r*32 + lane]
// (conflict-free); the group leader (q == 0) then adds them in stump order, which keeps the
// exact fp32 sequence of the definition (oracle c8).  The returned sum is valid in the leader.
template <int MC, int LC>
__device__ __forceinline__ float group_stage_mc(const uint32_t* __restrict__ T, int b, float nf, const GlobalRec& rec,
                                                int first, int n, int lg, bool act, float* lv, int lane) {
    const int gl = 1 << lg, q = lane & (gl - 1), g0 = lane & ~(gl - 1);
    float sum = 0.0f;
    for (int c0 = 0; c0 < n; c0 += gl * LC) {
        if (act) {
            float l[LC];
#pragma unroll
            for (int r = 0; r < LC; ++r) {
                const int j = c0 + q + (r << lg);
                l[r] = j < n ? eval_stump_mc<MC>(T, b, nf, rec, first + j) : 0.0f;
            }
#pragma unroll
            for (int r = 0; r < LC; ++r) lv[r * 32 + lane] = l[r];
        }
        __syncwarp();
        if (act && q == 0) {
            const int cn = min(gl * LC, n - c0);
#pragma unroll 8
            for (int j = 0; j < cn; ++j) sum = __fadd_rn(sum, lv[(j >> lg) * 32 + g0 + (j & (gl - 1))]);
        }
        __syncwarp();
    }
    return sum;
}

template <int LC>
__device__ __forceinline__ float group_stage(const uint32_t* __restrict__ T, int b, float nf, const GlobalRec& rec,
                                             int first, int n, int mc, int lg, bool act, float* lv, int lane) {
    if (mc <= 6) return group_stage_mc<6, LC>(T, b, nf, rec, first, n, lg, act, lv, lane);
    if (mc <= 8) return group_stage_mc<8, LC>(T, b, nf, rec, first, n, lg, act, lv, lane);
    if (mc <= 9) return group_stage_mc<9, LC>(T, b, nf, rec, first, n, lg, act, lv, lane);
    return group_stage_mc<MAX_CORNERS, LC>(T, b, nf, rec, first, n, lg, act, lv, lane);
}

// Dense first stage: each thread owns WPT windows of one column (stride STEP*TW words in
// shared memory).  The corner count nc is warp-uniform; common counts get a fully unrolled,
// branch-free body.
template <int NC, int WPT, int STRIDE>
__device__ __forceinline__ void dense_corners(const uint32_t* __restrict__ T, int base, const uint4& c0, const uint4& c1,
                                              const uint4& c2, int nc, uint32_t* f) {
#pragma unroll
    for (int c = 0; c < (NC > 0 ? NC : MAX_CORNERS); ++c) {
        if (NC > 0 || c < nc) {
            const int w = corner_word(c0, c1, c2, c);
            const uint32_t coef = (uint32_t)(w >> 16);
            const uint32_t* src = reinterpret_cast<const uint32_t*>(reinterpret_cast<const char*>(T + base) + (w & 0xffff));
#pragma unroll
            for (int i = 0; i < WPT; ++i) f[i] += coef * src[i * STRIDE];
        }
    }
}

template <int WPT, int STRIDE, class R>
__device__ __forceinline__ void dense_stage(const uint32_t* __restrict__ T, int base, const float* nf, float* sm,
                                            const R& rec, int first, int n) {
    for (int j = first; j < first + n; ++j) {
        const uint4 h = rec(4 * j);
        const uint4 c0 = rec(4 * j + 1), c1 = rec(4 * j + 2), c2 = rec(4 * j + 3);
        const int nc = (int)h.x;
        uint32_t f[WPT];
#pragma unroll
        for (int i = 0; i < WPT; ++i) f[i] = 0;
        switch (nc) {      // Table I features compile to 6 (edge), 8 (line, centre) or 9 (diagonal) corners
            case 6: dense_corners<6, WPT, STRIDE>(T, base, c0, c1, c2, nc, f); break;
            case 8: dense_corners<8, WPT, STRIDE>(T, base, c0, c1, c2, nc, f); break;
            case 9: dense_corners<9, WPT, STRIDE>(T, base, c0, c1, c2, nc, f); break;
            default: dense_corners<0, WPT, STRIDE>(T, base, c0, c1, c2, nc, f); break;
        }
        const float th = __int_as_float((int)h.y), lf = __int_as_float((int)h.z), rt = __int_as_float((int)h.w);
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const float tt = __fmul_rn(th, nf[i]);
            sm[i] = __fadd_rn(sm[i], (__int2float_rn((int)f[i]) < tt) ? lf : rt);
        }
    }
}

}  // namespace fdk
