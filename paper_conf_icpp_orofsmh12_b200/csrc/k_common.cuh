// k_common.cuh -- device helpers shared by the K2 cascade kernels (k_cascade.cu, k_tail.cu, k_soft.cu):
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

__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, int x, int y, int z, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
            smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar))
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

// Certified stage decision for warp-cooperative evaluation (GL lanes per window).  The
// definition (oracle c8) adds the n leaves sequentially in fp32; a cooperative evaluation gets
// the same leaves spread over lanes and adds them as a tree: per-lane sequential sums of c
// leaves, then lg butterfly levels (depth d = c - 1 + lg; every lane of the group ends with the
// same value).  Recursive summation of n terms satisfies |seq - S| <= gamma_{n-1} A and a tree of
// depth d |tree - S| <= gamma_d A (A = sum |leaf|, gamma_m = m u / (1 - m u), u = 2^-24;
// Higham, Accuracy and Stability of Numerical Algorithms, 2nd ed., 4.2), and the tree sum Ahat
// of |leaf| bounds A <= Ahat / (1 - gamma_d).  So |seq - tree| <= (n + d) u Ahat (1 + O(nu)),
// and B = (n + d + 2) * 2u * Ahat (+ 2^-100 absolute, for subnormal leaves) covers it with a 2x
// margin that also absorbs the rounding of B and of (tree - T).  If tree - T > B the sequential
// sum is >= T (pass); if T - tree > B it is < T (fail): the decision is the definition's.  Only
// when neither holds (|tree - T| <= B, a near tie) does the caller recompute the sequential sum.
// Returns 1 = pass, 0 = fail, -1 = undecided.
__device__ __forceinline__ int certify(float acc, float aacc, int n, int d, float T) {
    const float B = __fadd_rn(__fmul_rn(aacc, __fmul_rn(__int2float_rn(n + d + 2), 0x1p-23f)), 0x1p-100f);
    const float diff = __fsub_rn(acc, T);
    return diff > B ? 1 : (__fsub_rn(T, acc) > B ? 0 : -1);
}

// Tree-summed stage for a group of GL = 2^lg lanes per window: lane q evaluates stumps
// q, q + GL, ... (four in flight), keeps the sum and the sum of magnitudes of its leaves, then
// the group combines them with lg butterfly levels.  *d_out = tree depth (for certify).
template <int MC, class R>
__device__ __forceinline__ void group_stage_tree(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int first,
                                                 int n, int lg, bool act, int lane, float& acc, float& aacc) {
    const int gl = 1 << lg, q = lane & (gl - 1);
    acc = 0.0f;
    aacc = 0.0f;
    if (act) {
        int j = q;
        for (; j + 3 * gl < n; j += 4 * gl) {
            const float l0 = eval_stump_mc<MC>(T, b, nf, rec, first + j);
            const float l1 = eval_stump_mc<MC>(T, b, nf, rec, first + j + gl);
            const float l2 = eval_stump_mc<MC>(T, b, nf, rec, first + j + 2 * gl);
            const float l3 = eval_stump_mc<MC>(T, b, nf, rec, first + j + 3 * gl);
            acc = __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(acc, l0), l1), l2), l3);
            aacc = __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(aacc, fabsf(l0)), fabsf(l1)), fabsf(l2)), fabsf(l3));
        }
        for (; j < n; j += gl) {
            const float l = eval_stump_mc<MC>(T, b, nf, rec, first + j);
            acc = __fadd_rn(acc, l);
            aacc = __fadd_rn(aacc, fabsf(l));
        }
    }
    for (int o = gl >> 1; o > 0; o >>= 1) {
        acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, o));
        aacc = __fadd_rn(aacc, __shfl_xor_sync(0xffffffffu, aacc, o));
    }
}

template <class R>
__device__ __forceinline__ void group_stage_tree_mc(const uint32_t* __restrict__ T, int b, float nf, const R& rec,
                                                    int first, int n, int mc, int lg, bool act, int lane, float& acc,
                                                    float& aacc) {
    if (mc <= 6) return group_stage_tree<6>(T, b, nf, rec, first, n, lg, act, lane, acc, aacc);
    if (mc <= 8) return group_stage_tree<8>(T, b, nf, rec, first, n, lg, act, lane, acc, aacc);
    if (mc <= 9) return group_stage_tree<9>(T, b, nf, rec, first, n, lg, act, lane, acc, aacc);
    return group_stage_tree<MAX_CORNERS>(T, b, nf, rec, first, n, lg, act, lane, acc, aacc);
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
