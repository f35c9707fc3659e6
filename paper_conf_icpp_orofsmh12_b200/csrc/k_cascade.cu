// k_cascade.cu -- K2: persistent cascade evaluator over every window of every pyramid level.
//
// Paper: each integral image is cut into n x m chunks, one thread block per
// chunk, one thread per window; each block stages its chunk (2n x 2m values, eqs. 1-4) in
// shared memory, then every thread walks the stages with early exit; feature attributes sit
// in constant memory for warp-uniform broadcast.  B200 design:
//   * one persistent launch covers every (frame, level, tile) of a frame group -- replaces
//     the paper's one-kernel-per-scale streams;
//   * a tile of TX x TY windows needs a (TX+24) x (TY+24) block of ii and sqii: one 4-D TMA
//     (cp.async.bulk.tensor) per tile completing on an mbarrier (optionally double buffered);
//   * stump records of the first stages live in the kernel-parameter constant bank, so the
//     warp-uniform record reads go through the uniform datapath (the paper's constant-memory
//     broadcast); each Haar feature is pre-compiled on the host into its distinct
//     integral-image corners with integer coefficients (sum_r wt_r*R_r == sum_c coef_c*ii_c
//     exactly, mod 2^32);
//   * stage 1 (94.5% of windows stop there) is evaluated densely, each thread
//     owning WPT windows of a column; survivors are compacted with warp ballots into a
//     shared-memory queue after every stage so deeper stages run on full warps (the
//     divergence problem of P:L1228-1258); when few windows survive, GL lanes share a window
//     (one stump per lane) and the leaves are added in stump order;
//   * fp32 arithmetic matches the oracle bit for bit: __fmul_rn/__fadd_rn (no FMA
//     contraction), __int2float_rn, __ll2float_rn, IEEE __fsqrt_rn.
// Kernels: k_stage1 + k_deepq (k_deepq.cuh) or k_deep1 (split at stage 2), k_f1 (+ k_deep1<F1>:
// SURVEY 8(f) f1, tile-local integrals built in shared memory).  (A fused kernel running every
// stage of a tile in one CTA was measured slower in rounds 1-2 and removed.)
// This file is also compiled at run time by NVRTC with the cascade's specialised stages
// (fd_jit.cpp: FD_JIT_STAGE1, FD_JIT_DEEP, FD_PACKED_WORDS).
#include "k_common.cuh"

namespace fdk {

#if defined(FD_K2_TIMING) && !defined(__CUDACC_RTC__)
// [0] tiles, [1] TMA-wait cycles, [2] stage-1 cycles, [3] deep-stage cycles, [4+s] tiles whose
// deepest stage loop ended at s, [16+s] cycles of deep stage s (block-wide loop iteration),
// [48+s] tiles that ran deep stage s, [80] tail cycles, [81] tails, [82] mode-M cycles,
// [83] mode-L cycles (diagnostic build only: -DFD_K2_TIMING)
__device__ unsigned long long g_k2_timing[128];
extern "C" int fd_debug_k2_timing(unsigned long long* out, int reset) {
    if (cudaMemcpyFromSymbol(out, g_k2_timing, sizeof(g_k2_timing)) != cudaSuccess) return -1;
    if (reset) {
        unsigned long long z[128] = {};
        cudaMemcpyToSymbol(g_k2_timing, z, sizeof(z));
    }
    return 0;
}
#endif

#ifndef FD_JIT_DEEP
#define FD_JIT_DEEP 0        // run-time specialised kernel: deep stages [1, FD_JIT_DEEP) are generated code
#endif

#ifdef FD_PACKED_WORDS
// f3 (reading R13): the cascade's compressed records, resident in this program's
// constant bank (58 KB for the 2913-stump c6q) and read warp-uniformly (constant-cache broadcast,
// the paper's reason for compressing them).  Record j: words 0-2 = rectangles (x | y<<5 | w<<10 in
// the low 16 bits, h | wt<<5 in the high 16 bits, wt 6-bit two's complement; an absent rectangle
// is all zeros), word 3 = theta | left << 16, word 4 = right | nrect << 16 (binary16 values).
__constant__ uint32_t fd_pk[FD_PACKED_WORDS];

// binary16 -> binary32, exact (finite values only: the parser refuses the others): a normal value
// re-biases its exponent (15 -> 127); a subnormal m * 2^-24 is an exact fp32 product
__device__ __forceinline__ float half_bits_to_float(uint32_t h) {
    const uint32_t sgn = (h & 0x8000u) << 16, e = (h >> 10) & 31u, m = h & 1023u;
    if (e) return __uint_as_float(sgn | ((e + 112u) << 23) | (m << 13));
    const float v = __fmul_rn(__uint2float_rn(m), 0x1p-24f);
    return sgn ? -v : v;
}

// One stage for one window from the compressed records: f = sum_r wt_r * (A - B - C + D) (mod 2^32,
// equal to the corner-compiled sum), leaf = ((float)f < theta*nf) ? left : right, fp32 sum in
// stump order (oracle c6-c8).
template <int STEP>
__device__ __forceinline__ float eval_stage_packed(const uint32_t* __restrict__ T, int b, float nf, int first, int n) {
    constexpr int TW = tile_w(STEP);
    float sum = 0.0f;
    for (int j = first; j < first + n; ++j) {
        const uint32_t* r = fd_pk + FD_PK_WORDS * j;
        const uint32_t w3 = r[3], w4 = r[4];
        const int nr = (int)(w4 >> 16);
        uint32_t f = 0;
#pragma unroll
        for (int q = 0; q < 3; ++q) {
            if (q < nr) {
                const uint32_t w = r[q];
                const int x = (int)(w & 31u), y = (int)((w >> 5) & 31u), ww = (int)((w >> 10) & 31u);
                const int h = (int)((w >> 16) & 31u), wt = (int)(w << 5) >> 26;
                const uint32_t* a = T + b + y * TW + x;
                const uint32_t R = a[0] - a[ww] - a[h * TW] + a[h * TW + ww];
                f += (uint32_t)wt * R;
            }
        }
        const float th = half_bits_to_float(w3 & 0xffffu), lf = half_bits_to_float(w3 >> 16);
        const float rt = half_bits_to_float(w4 & 0xffffu);
        sum = __fadd_rn(sum, (__int2float_rn((int)f) < __fmul_rn(th, nf)) ? lf : rt);
    }
    return sum;
}
#endif

// Output of a window of ii slot sl (batch tile table in shared memory).
template <int STEP, bool DEPTH>
struct WinOut {
    const CascadeParams& p;
    const int *frame, *lvl, *wx0, *wy0;
    static constexpr int TX = k2_tx(STEP);
    __device__ __forceinline__ long long index(int sl, int idx) const {
        const int k = lvl[sl];
        return (long long)frame[sl] * p.win_per_frame + __ldg(&p.lv[k].win0) +
               (long long)(wy0[sl] + idx / TX) * __ldg(&p.lv[k].nx) + (wx0[sl] + idx % TX);
    }
    // a window that passed every stage (depth N): detection record or depth/score map entry
    __device__ __forceinline__ void emit(int sl, int idx, float score) const {
        if (p.stage_counts) atomicAdd(p.stage_counts + p.n_stages, 1ull);
        if (DEPTH) {
            const long long o = index(sl, idx);
            p.depth[o] = (uint8_t)(p.n_stages < 255 ? p.n_stages : 255);
            p.score[o] = score;
        } else {
            const unsigned long long at = atomicAdd(p.det_count, 1ull);
            if ((long long)at < p.det_cap) {
                p.det_keys[at] = det_key(frame[sl], lvl[sl], (wy0[sl] + idx / TX) * STEP, (wx0[sl] + idx % TX) * STEP);
                p.det_scores[at] = score;
            }
        }
    }
    // depth mode: the window stopped at stage s (depth s) with stage sum `score`
    __device__ __forceinline__ void reject(int sl, int idx, int s, float score) const {
        if (DEPTH) {
            const long long o = index(sl, idx);
            p.depth[o] = (uint8_t)(s < 255 ? s : 255);
            p.score[o] = score;
        }
    }
};

// One window finished by one warp from stage s on (tail queue full or absent): lane j evaluates
// stump c0 + j, the leaves are added in stump order (independent shuffles, serial adds -- the
// definition's fp32 sequence), early exit on the first failed stage.
template <int STEP, bool DEPTH>
__device__ __noinline__ void finish_window_warp(const CascadeParams& p, const uint32_t* __restrict__ slots, int b,
                                                float nfw, int s, int sl, int idx, const WinOut<STEP, DEPTH>& out) {
    const int lane = threadIdx.x & 31, N = p.n_stages;
    const GlobalRec grec{p.stumps};
    int s2 = s;
    float sum = 0.0f;
    for (; s2 < N; ++s2) {
        StageDev sd;
        if (s2 < p.n_pstages) {
            sd.first = p.pstages[s2].first;
            sd.n = p.pstages[s2].n;
            sd.T = p.pstages[s2].T;
            sd.mc = p.pstages[s2].mc;
        } else {
            sd = p.stages[s2];
        }
        if (s2 > s && lane == 0 && p.stage_counts) atomicAdd(p.stage_counts + s2, 1ull);
        sum = 0.0f;
        for (int c0 = 0; c0 < sd.n; c0 += 32) {
            const int j = c0 + lane;
            float leaf = 0.0f;
            if (j < sd.n) leaf = eval_stage(slots, b, nfw, grec, sd.first + j, 1, sd.mc);
            const int m = min(32, sd.n - c0);
#pragma unroll
            for (int t2 = 0; t2 < 32; ++t2) {
                const float v = __shfl_sync(0xffffffffu, leaf, t2);
                if (t2 < m) sum = __fadd_rn(sum, v);
            }
        }
        if (!(sum >= sd.T)) break;
    }
    if (lane == 0) {
        if (s2 < N)
            out.reject(sl, idx, s2, sum);
        else
            out.emit(sl, idx, sum);
    }
}

// Deep stages (1 .. N-1) over a pool of stage-1 survivors held in shared memory: entry e has
// ploc[e] = slot << 11 | window index (within the slot's tile) and nf pnf[e]; s_cnt[s0 % 3] = pool
// size (the other two 0) on entry; the pool enters stage s0.  Stage-synchronous: each stage's survivors are
// ballot-compacted into the other list and the block synchronises once per stage.  Lane per
// window (uniform stump records) while windows are plentiful, GL lanes per window (tree sum +
// certified decision) when fewer than lane_min remain, and once at most tail_n are left they go
// to the global tail queue (k_tail.cu) -- or, when it is full or absent, are finished here one
// warp per window.  Ends with a block barrier.
// Barrier over the threads running a phase: the whole CTA (BAR = 0) or the named barrier BAR
// over THREADS threads (a warp group of a warp-specialised kernel).
template <int BAR, int THREADS>
__device__ __forceinline__ void phase_sync() {
    if constexpr (BAR == 0)
        __syncthreads();
    else
        asm volatile("bar.sync %0, %1;" ::"n"(BAR), "n"(THREADS) : "memory");
}

// Split-stump partial sums: the stumps first + q, first + q + wpb, ... of a stage for one window
// (sequential fp32 sums of the leaves and of their magnitudes); records warp-uniform.
template <int MC, class R>
__device__ __forceinline__ void split_partial(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int first,
                                              int n, int q, int wpb, float& acc, float& aacc) {
    for (int j = q; j < n; j += wpb) {
        const float l = eval_stump_mc<MC>(T, b, nf, rec, first + j);
        acc = __fadd_rn(acc, l);
        aacc = __fadd_rn(aacc, fabsf(l));
    }
}
template <class R>
__device__ __forceinline__ void split_partial_mc(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int first,
                                                 int n, int mc, int q, int wpb, float& acc, float& aacc) {
    if (mc <= 6) return split_partial<6>(T, b, nf, rec, first, n, q, wpb, acc, aacc);
    if (mc <= 8) return split_partial<8>(T, b, nf, rec, first, n, q, wpb, acc, aacc);
    if (mc <= 9) return split_partial<9>(T, b, nf, rec, first, n, q, wpb, acc, aacc);
    return split_partial<MAX_CORNERS>(T, b, nf, rec, first, n, q, wpb, acc, aacc);
}

// red: THREADS / 32 x 32 float2 of shared memory for the split-stump mode (nullptr: not used)
template <int STEP, bool DEPTH, int CP, int THREADS = k2_threads(STEP), int TID0 = 0, int BAR = 0>
__device__ __forceinline__ void deep_phase(const CascadeParams& p, int s0, const uint32_t* __restrict__ slots,
                                           const float* pnf, const uint16_t* ploc, uint16_t* lists, int* s_cnt,
                                           int& s_tpos, const WinOut<STEP, DEPTH>& out, float2* red = nullptr) {
    constexpr int TX = k2_tx(STEP), TW = tile_w(STEP), PBUF = k2_pbuf(STEP);
    const int tid = (int)threadIdx.x - TID0, warp = tid >> 5, lane = tid & 31;
    const int lane_min = min(p.lane_min, THREADS / 2 + 1);
    const int N = p.n_stages;
    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};
    const int tail_n = p.tail_q ? p.tail_n : THREADS / 32;
    const int* s_frame = out.frame;
    const int* s_lvl = out.lvl;
    const int* s_wx0 = out.wx0;
    const int* s_wy0 = out.wy0;
    auto emit = [&](int sl, int idx, float score) { out.emit(sl, idx, score); };
    auto reject = [&](int sl, int idx, int s, float score) { out.reject(sl, idx, s, score); };
#ifdef FD_K2_TIMING
    const long long tm2 = clock64();
#endif
    int s = s0;
    // one deep stage; sd is a parameter-bank (uniform) or global stage descriptor.  Stage s0's
    // input is the pool itself (entry e), later stages read pool indices from lists.
    auto deep_stage = [&](const StageDev& sd, int n) {
        const uint16_t* lin = lists + (s & 1) * CP;
        uint16_t* lout = lists + ((s + 1) & 1) * CP;
        const bool last = s == N - 1;
        // stages [1, FD_JIT_DEEP) of the run-time specialised kernel: immediate-offset code,
        // always one lane per window
        const bool jit_s = FD_JIT_DEEP > 0 && s < FD_JIT_DEEP;
        if (red && n <= p.split_max && n <= 2 * 32 && THREADS >= 64) {
            // split-stump mode (few windows): lanes = windows (blocks of 32), the WARPS / nb warps
            // of a block each evaluate every wpb-th stump of the stage for all the block's
            // windows with warp-uniform records, so a stage costs ~n_s / wpb stump evaluations of
            // latency instead of n_s.  The partial sums are added in a fixed order (q = 0, 1, ..)
            // and the decision is certified against the rounding bound of that summation tree
            // (k_common.cuh certify: leaf depth <= ceil(n_s / wpb) - 1 + wpb - 1); near ties and
            // output scores are recomputed with the definition's sequential sum.
            constexpr int WARPS = THREADS / 32;
            const int nb = (n + 31) >> 5;
            const int wpb = WARPS / nb;
            const int bk = warp / wpb, q = warp - bk * wpb;
            const int e = bk * 32 + lane;
            const bool act = bk < nb && e < n;
            int pe = 0, sl = 0, idx = 0, b = 0;
            float nfw = 1.0f;
            if (act) {
                pe = s == s0 ? e : lin[e];
                const int loc = ploc[pe];
                sl = loc >> 11;
                idx = loc & 2047;
                b = sl * PBUF + (idx / TX) * STEP * TW + (idx % TX) * STEP;
                nfw = pnf[pe];
            }
            const bool in_param = sd.first + sd.n <= p.n_pstumps;
            float acc = 0.0f, aacc = 0.0f;
            if (act) {
                if (in_param)
                    split_partial_mc(slots, b, nfw, prec, sd.first, sd.n, sd.mc, q, wpb, acc, aacc);
                else
                    split_partial_mc(slots, b, nfw, grec, sd.first, sd.n, sd.mc, q, wpb, acc, aacc);
            }
            red[warp * 32 + lane] = make_float2(acc, aacc);
            phase_sync<BAR, THREADS>();
            if (act && q == 0) {
                float t = 0.0f, ta = 0.0f;
                for (int r = 0; r < wpb; ++r) {
                    const float2 v = red[(bk * wpb + r) * 32 + lane];
                    t = __fadd_rn(t, v.x);
                    ta = __fadd_rn(ta, v.y);
                }
                int dec = certify(t, ta, sd.n, (sd.n + wpb - 1) / wpb + wpb, sd.T);
                float sum = t;
                if (dec < 0 || (dec == 1 && last) || (DEPTH && dec == 0)) {
                    sum = in_param ? eval_stage(slots, b, nfw, prec, sd.first, sd.n, sd.mc)
                                   : eval_stage(slots, b, nfw, grec, sd.first, sd.n, sd.mc);
                    dec = sum >= sd.T ? 1 : 0;
                }
                if (dec == 1) {
                    if (last)
                        emit(sl, idx, sum);
                    else
                        lout[atomicAdd(&s_cnt[(s + 1) % 3], 1)] = (uint16_t)pe;
                } else {
                    reject(sl, idx, s, sum);
                }
            }
            return;
        }
        if (!jit_s && n < lane_min) {
            // fewer windows than half the block: GL = 2^lg lanes per window (the largest
            // power of two with n*GL <= THREADS, so one pass covers every window and
            // all warps work); the group's lanes evaluate different stumps, the leader adds
            // the leaves in stump order (the exact fp32 sequence of the definition).
            int lg = 1;
            while (lg < 5 && (n << (lg + 1)) <= THREADS) ++lg;
            const int e = tid >> lg;
            const bool act = e < n;
            const int pe = act ? (s == s0 ? e : lin[e]) : 0;
            const int loc = act ? ploc[pe] : 0;
            const int sl = loc >> 11, idx = loc & 2047;
            const int b = sl * PBUF + (idx / TX) * STEP * TW + (idx % TX) * STEP;
            const float nfw = act ? pnf[pe] : 1.0f;
            // tree sum + certified decision; the sequential sum only where the decision is a
            // near tie or the score is an output (accepted window, depth-mode rejection)
            float acc, aacc;
            group_stage_tree_mc(slots, b, nfw, grec, sd.first, sd.n, sd.mc, lg, act, lane, acc, aacc);
            int dec = certify(acc, aacc, sd.n, (sd.n + (1 << lg) - 1) / (1 << lg) - 1 + lg, sd.T);
            float sum = acc;
            const bool need = act && (dec < 0 || (dec == 1 && last) || (DEPTH && dec == 0));
#ifdef FD_K2_TIMING
            if (act && (lane & ((1 << lg) - 1)) == 0) {
                atomicAdd(&g_k2_timing[95], 1ull);
                if (dec < 0) atomicAdd(&g_k2_timing[94], 1ull);
                if (need) atomicAdd(&g_k2_timing[96], 1ull);
            }
#endif
            if (need && (lane & ((1 << lg) - 1)) == 0) {
                // rare: the group leader adds the leaves itself, in stump order
                // (records from global memory: a divergent constant-bank read serialises)
                sum = eval_stage(slots, b, nfw, grec, sd.first, sd.n, sd.mc);
                dec = sum >= sd.T ? 1 : 0;
            }
            if (act && (lane & ((1 << lg) - 1)) == 0) {
                if (dec == 1) {
                    if (last)
                        emit(sl, idx, sum);
                    else
                        lout[atomicAdd(&s_cnt[(s + 1) % 3], 1)] = (uint16_t)pe;
                } else {
                    reject(sl, idx, s, sum);
                }
            }
            return;
        }
        const bool in_param = sd.first + sd.n <= p.n_pstumps;
        for (int e0 = warp * 32; e0 < n; e0 += THREADS) {
            const int e = e0 + lane;
            const bool act = e < n;
            int pe = 0, sl = 0, idx = 0;
            float sum = 0.0f;
            if (act) {
                pe = s == s0 ? e : lin[e];
                const int loc = ploc[pe];
                sl = loc >> 11;
                idx = loc & 2047;
                const int b = sl * PBUF + (idx / TX) * STEP * TW + (idx % TX) * STEP;
                const float nfw = pnf[pe];
#if FD_JIT_DEEP > 0
                if (jit_s)
                    sum = jit_deep(s, slots + b, nfw);
                else
#endif
#ifdef FD_PACKED_WORDS
                    sum = eval_stage_packed<STEP>(slots, b, nfw, sd.first, sd.n);   // f3: constant-bank records
#else
                    sum = in_param ? eval_stage(slots, b, nfw, prec, sd.first, sd.n, sd.mc)
                                   : eval_stage(slots, b, nfw, grec, sd.first, sd.n, sd.mc);
#endif
            }
            const bool pass = act && (sum >= sd.T);
            if (act && !pass) reject(sl, idx, s, sum);
            if (last) {
                if (pass) emit(sl, idx, sum);
                continue;
            }
            const unsigned m = __ballot_sync(0xffffffffu, pass);
            if (m) {
                int pos = 0;
                if (lane == 0) pos = atomicAdd(&s_cnt[(s + 1) % 3], __popc(m));
                pos = __shfl_sync(0xffffffffu, pos, 0);
                if (pass) lout[pos + __popc(m & ((1u << lane) - 1u))] = (uint16_t)pe;
            }
        }
    };
    for (; s < N; ++s) {
#ifdef FD_K2_TIMING
        const long long ts0 = clock64();
#endif
        const int n = s_cnt[s % 3];
        if (tid == 0 && p.stage_counts && n) atomicAdd(p.stage_counts + s, (unsigned long long)n);
        if (n == 0) break;
        if ((n <= tail_n && !(FD_JIT_DEEP > 0 && s < FD_JIT_DEEP)) || (s >= p.s_tail && p.tail_q)) {
            // tail: few windows left.  They go to the global tail queue (finished by
            // k_tail, one warp per window) so this CTA moves on to its next tiles instead of
            // waiting for its deepest window; whatever does not fit in the queue is finished
            // here, one warp per window.
            const uint16_t* lin = lists + (s & 1) * CP;
            if (tid == 0) s_tpos = p.tail_q ? (int)atomicAdd(p.tail_count, (unsigned)n) : p.tail_cap;
            phase_sync<BAR, THREADS>();
            const int tpos = s_tpos;
            for (int e = tid; e < n && tpos + e < p.tail_cap; e += THREADS) {
                const int pe = s == s0 ? e : lin[e];
                const int loc = ploc[pe];
                const int sl = loc >> 11, idx = loc & 2047;
                uint4 q;
                q.x = ((unsigned)s_lvl[sl] << 8) | (unsigned)s;
                q.y = ((unsigned)(s_wy0[sl] + idx / TX) << 16) | (unsigned)(s_wx0[sl] + idx % TX);
                q.z = (unsigned)__float_as_int(pnf[pe]);
                q.w = (unsigned)(s_frame[sl] - p.frame_base);
                p.tail_q[tpos + e] = q;
            }
            for (int e = warp; e < n; e += THREADS / 32) {
                if (tpos + e < p.tail_cap) continue;
                const int pe = s == s0 ? e : lin[e];
                const int loc = ploc[pe];
                const int sl = loc >> 11, idx = loc & 2047;
                const int b = sl * PBUF + (idx / TX) * STEP * TW + (idx % TX) * STEP;
                finish_window_warp<STEP, DEPTH>(p, slots, b, pnf[pe], s, sl, idx, out);
            }
#ifdef FD_K2_TIMING
            if (tid == 0) {
                atomicAdd(&g_k2_timing[80], (unsigned long long)(clock64() - ts0));
                atomicAdd(&g_k2_timing[81], (unsigned long long)n);
            }
#endif
            break;
        }
        if (tid == 0) s_cnt[(s + 2) % 3] = 0;
        {
            StageDev sd;                  // one call site keeps deep_stage inlined
            if (s < p.n_pstages) {
                sd.first = p.pstages[s].first;
                sd.n = p.pstages[s].n;
                sd.T = p.pstages[s].T;
                sd.mc = p.pstages[s].mc;
            } else {
                sd = p.stages[s];
            }
            deep_stage(sd, n);
        }
        phase_sync<BAR, THREADS>();
#ifdef FD_K2_TIMING
        if (tid == 0) {
            const unsigned long long dt = (unsigned long long)(clock64() - ts0);
            const int si = s < 32 ? s : 31;
            atomicAdd(&g_k2_timing[16 + si], dt);
            atomicAdd(&g_k2_timing[48 + si], 1ull);
            atomicAdd(&g_k2_timing[n < lane_min ? 82 : 83], dt);
        }
#endif
    }
#ifdef FD_K2_TIMING
    if (tid == 0) {
        atomicAdd(&g_k2_timing[3], (unsigned long long)(clock64() - tm2));
        atomicAdd(&g_k2_timing[4 + (s < 11 ? s : 11)], 1ull);
        atomicAdd(&g_k2_timing[84], 1ull);
    }
#endif
    phase_sync<BAR, THREADS>();
}

// Tile number tn of a frame group -> frame (global), level, window origin, TMA coordinates.
struct TileAt {
    int g, k, wx0, wy0, x, y;
};
template <int STEP>
__device__ __forceinline__ TileAt tile_at(const CascadeParams& p, int tn) {
    TileAt t;
    t.g = tn / p.tiles_per_frame;
    const int r = tn % p.tiles_per_frame;
    int k = 0;
    while (k + 1 < p.n_levels && __ldg(&p.lv[k + 1].tile0) <= r) ++k;
    const int tl = r - __ldg(&p.lv[k].tile0);
    const int tx = __ldg(&p.lv[k].tiles_x);
    t.k = k;
    t.wx0 = (tl % tx) * k2_tx(STEP);
    t.wy0 = (tl / tx) * k2_ty(STEP);
    t.x = t.wx0 * STEP;
    t.y = t.wy0 * STEP;
    return t;
}

// ======================================================================== split K2, kernel a
// k_stage1: the dense first stage and the second stage, the throughput part of the cascade
// (c3: 10 of the 11.8 stumps per window, 94.5% of windows stop at stage 1, 71% of the rest at
// stage 2).  Persistent over every (frame, level, tile) of the group:
//   * the tile's ii and sqii planes arrive by TMA; the variance normalisation (oracle c5) reads
//     sqii, after which the NEXT tile is claimed and its ii (into the other ii buffer) and sqii
//     (into the now dead sqii plane) are fetched while this tile's stages run;
//   * stage 1 is evaluated densely (WPT windows per thread down a column, run-time specialised
//     code for step 1) and its survivors ballot-compacted into a shared list;
//   * stage 2 (p.s0 == 2) runs over that list one lane per window; the survivors of the last
//     stage run here -- window index and nf -- go to a global list at an offset reserved per tile
//     (tile_rec[tile] = (offset, count)) for k_deep1.
template <int STEP, bool DEPTH>
__device__ __forceinline__ void stage1_tiles(const CascadeParams& p, uint8_t* smem_raw) {
    using G = TileGeoA<STEP>;
    constexpr int TW = tile_w(STEP), TX = k2_tx(STEP), TY = k2_ty(STEP), WPT = k2_wpt(STEP);
    constexpr int WARPS_X = TX / 32, PLANE = tile_w(STEP) * tile_h(STEP), THREADS = k2_threads(STEP);
    uint32_t* Q = reinterpret_cast<uint32_t*>(smem_raw + G::OFF_Q);           // sqii plane (mod 2^32)
    float* snf = reinterpret_cast<float*>(smem_raw + G::OFF_SNF);             // [NW] stage-1 survivors: nf
    uint16_t* sidx = reinterpret_cast<uint16_t*>(smem_raw + G::OFF_SIDX);    //       and window index
    __shared__ __align__(8) uint64_t mbar[2];
    __shared__ int s_tile[2], s_frame[2], s_lvl[2], s_wx0[2], s_wy0[2];
    __shared__ int s_c1[2], s_c2[2], s_off, s_prev, s_prev_off;   // survivor counters per parity of the tile
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const StageDev& st0 = p.pstages[0];
    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};
    // tid 0: claim the next tile for ii buffer b and start its TMAs (ii -> buffer b, sqii -> Q)
    auto claim = [&](int b) {
        const int tn = (int)atomicAdd(p.tile_counter, 1u);
        s_tile[b] = tn;
        if (tn < p.total_tiles) {
            const TileAt t = tile_at<STEP>(p, tn);
            s_frame[b] = p.frame_base + t.g;
            s_lvl[b] = t.k;
            s_wx0[b] = t.wx0;
            s_wy0[b] = t.wy0;
            uint32_t* Tb = reinterpret_cast<uint32_t*>(smem_raw) + b * G::PBUF;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_expect_tx(&mbar[b], 2 * PLANE * 4);
            tma_load_4d(Tb, p.tmaps + t.k, t.x, t.y, 0, t.g, &mbar[b]);
            tma_load_4d(Q, p.tmaps + t.k, t.x, t.y, 1, t.g, &mbar[b]);
        }
    };
    // this thread's windows (the same for every tile): WPT windows of column lx from row ly0
    const int lx = lane + 32 * (warp % WARPS_X);
    const int ly0 = (warp / WARPS_X) * WPT;
    const int base = ly0 * STEP * TW + lx * STEP;
    // variance normalisation (oracle c5) of this thread's windows of the tile in ii buffer bb + Q
    auto variance = [&](int bb, float* nfo) {
        const uint32_t* Tb = reinterpret_cast<const uint32_t*>(smem_raw) + bb * G::PBUF;
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int bo = base + i * STEP * TW;
            const uint32_t S = Tb[bo + WIN * TW + WIN] - Tb[bo + WIN] - Tb[bo + WIN * TW] + Tb[bo];
            const uint32_t q = Q[bo + WIN * TW + WIN] - Q[bo + WIN] - Q[bo + WIN * TW] + Q[bo];
            const long long v = 576LL * (long long)q - (long long)S * (long long)S;
            nfo[i] = v > 0 ? __fsqrt_rn(__ll2float_rn(v)) : 1.0f;
        }
    };
    if (tid == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        s_prev = -1;
        s_c1[0] = s_c1[1] = s_c2[0] = s_c2[1] = 0;
        claim(0);
    }
    __syncthreads();
    uint32_t phases = 0;
    float nf[WPT];
    if (s_tile[0] < p.total_tiles) {              // the first tile's variance; later tiles' in the loop
        mbar_wait(&mbar[0], 0u);
        phases ^= 1u;
        variance(0, nf);
    }
    for (int it = 0;; ++it) {
        const int b = it & 1;
        __syncthreads();                          // (A) previous tile done: list, counters, its ii buffer and
                                                  //     (this tile's variance taken) the sqii buffer free
        const int tn = s_tile[b];
        if (tid == 0) {
            // the previous tile's record; its counters are reset for the tile after this one (a
            // barrier separates that reset from their next use)
            if (s_prev >= 0) {
                p.tile_rec[s_prev] = make_uint2((unsigned)s_prev_off, (unsigned)s_c2[b ^ 1]);
                if (p.tile_list && s_c2[b ^ 1] > 0)      // k_deepq's compact list of tiles with work
                    p.tile_list[atomicAdd(p.tile_list_count, 1u)] =
                        make_uint4((unsigned)s_prev, (unsigned)s_prev_off, (unsigned)s_c2[b ^ 1], 0u);
            }
            s_prev = -1;
            s_c1[b ^ 1] = 0;
            s_c2[b ^ 1] = 0;
        }
        if (tn >= p.total_tiles) break;
        if (tid == 0) claim(b ^ 1);               // prefetch: next ii -> the other buffer, next sqii -> Q
        const WinOut<STEP, DEPTH> out{p, s_frame + b, s_lvl + b, s_wx0 + b, s_wy0 + b};
        const uint32_t* T = reinterpret_cast<const uint32_t*>(smem_raw) + b * G::PBUF;
        const int k = s_lvl[b];
        const int nx = __ldg(&p.lv[k].nx), ny = __ldg(&p.lv[k].ny);
        const int wx0 = s_wx0[b], wy0 = s_wy0[b];
        const bool colok = wx0 + lx < nx;
        float sm[WPT];
#pragma unroll
        for (int i = 0; i < WPT; ++i) sm[i] = 0.0f;
#ifdef FD_JIT_STAGE1
        jit_stage1(T + base, nf, sm);
#else
        if (st0.first + st0.n <= p.n_pstumps)
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, prec, st0.first, st0.n);
        else
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, grec, st0.first, st0.n);
#endif
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int wy = wy0 + ly0 + i;
            const bool valid = colok && wy < ny;
            const bool pass = valid && (sm[i] >= st0.T);
            const int idx = (ly0 + i) * TX + lx;
            if (DEPTH && valid && !pass) out.reject(0, idx, 0, sm[i]);
            if (p.n_stages == 1) {
                if (pass) out.emit(0, idx, sm[i]);
                continue;
            }
            const unsigned m = __ballot_sync(0xffffffffu, pass);
            if (m) {
                int pos = 0;
                if (lane == 0) pos = atomicAdd(&s_c1[b], __popc(m));
                pos = __shfl_sync(0xffffffffu, pos, 0);
                if (pass) {
                    const int at = pos + __popc(m & ((1u << lane) - 1u));
                    sidx[at] = (uint16_t)idx;
                    snf[at] = nf[i];
                }
            }
        }
        __syncthreads();                          // (C) stage-1 survivor list complete
        const int c = s_c1[b];
        if (tid == 0) {
            // reserve c global entries for this tile's survivors (an upper bound after stage 2)
            s_off = c ? (int)atomicAdd(p.surv_count, (unsigned)c) : 0;
            if (p.stage_counts) {
                atomicAdd(p.stage_counts, (unsigned long long)min(TX, nx - wx0) * (unsigned long long)min(TY, ny - wy0));
                if (p.s0 == 2 && c) atomicAdd(p.stage_counts + 1, (unsigned long long)c);
            }
        }
        __syncthreads();                          // (D) offset visible
        const int off = s_off;
        if (p.s0 < 2 || p.n_stages < 2) {
            for (int e = tid; e < c; e += THREADS) p.surv[off + e] = make_uint2(sidx[e], (unsigned)__float_as_int(snf[e]));
            if (tid == 0) s_c2[b] = c;
        } else {
            // stage 2 over the list, one lane per window; survivors straight to the global list
            const StageDev& sd = p.pstages[1];
            const bool last = p.n_stages == 2;
            for (int e0 = warp * 32; e0 < c; e0 += THREADS) {
                const int e = e0 + lane;
                const bool act = e < c;
                int idx = 0;
                float nfw = 1.0f, sum = 0.0f;
                if (act) {
                    idx = sidx[e];
                    nfw = snf[e];
                    const int bo = (idx / TX) * STEP * TW + (idx % TX) * STEP;
#if FD_JIT_DEEP > 1
                    sum = jit_deep(1, T + bo, nfw);
#else
                    sum = sd.first + sd.n <= p.n_pstumps ? eval_stage(T, bo, nfw, prec, sd.first, sd.n, sd.mc)
                                                         : eval_stage(T, bo, nfw, grec, sd.first, sd.n, sd.mc);
#endif
                }
                const bool pass = act && (sum >= sd.T);
                if (act && !pass) out.reject(0, idx, 1, sum);
                if (last) {
                    if (pass) out.emit(0, idx, sum);
                    continue;
                }
                const unsigned m = __ballot_sync(0xffffffffu, pass);
                if (m) {
                    int pos = 0;
                    if (lane == 0) pos = atomicAdd(&s_c2[b], __popc(m));
                    pos = __shfl_sync(0xffffffffu, pos, 0);
                    if (pass)
                        p.surv[off + pos + __popc(m & ((1u << lane) - 1u))] =
                            make_uint2((unsigned)idx, (unsigned)__float_as_int(nfw));
                }
            }
        }
        // the next tile's variance: its ii and sqii planes arrive during this tile's stages, and
        // every thread takes its own windows' nf here -- the warps without stage-2 work first
        if (s_tile[b ^ 1] < p.total_tiles) {
            mbar_wait(&mbar[b ^ 1], (phases >> (b ^ 1)) & 1u);
            phases ^= 1u << (b ^ 1);
            variance(b ^ 1, nf);
        }
        if (tid == 0) {
            s_prev = tn;                          // tile_rec written after the next barrier (A)
            s_prev_off = off;
        }
    }
}

template <int STEP, bool DEPTH>
__global__ void __launch_bounds__(k2_threads(STEP), 3) k_stage1(const __grid_constant__ CascadeParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    stage1_tiles<STEP, DEPTH>(p, smem_raw);
}

// ======================================================================== f1: fused K2
// the tile's integral images are built in shared memory from its level pixels,
// so no ii / sqii plane ever makes an HBM round trip (the paper's integral kernels take "20% of
// the total" time; P:L368-384 scan + transpose).  The level pixels of a tile's
// (TW-1) x (TH-1) region arrive as one 3-D TMA box (u8, 5.3 KB at step 1, double buffered so the
// next tile's box is in flight while this tile is evaluated).
//
// Tile-local integral (reading R4: every rectangle sum is a difference of four ii values, so the
// origin of the integral does not matter; tile-local sums are < 2^32, so u32 is exact):
//   row pass    thread (r, s) owns pixel row r, columns [s*SEGW, (s+1)*SEGW): it sums its segment,
//               the NSEG segments of a row (adjacent lanes) exchange exclusive offsets with
//               shuffles, then it writes running row prefixes of p and p^2 into rows 1.. of T / Q;
//   column pass thread per (column, plane) adds down the TH-1 rows (loads batched 8 at a time).
// Row 0 and column 0 of both planes are zero.  Ends with a block barrier.
// THREADS: block size; WITH_Q: also build the sqii plane (k_f1; k_deep1 rebuilds ii only)
template <int STEP, int THREADS = k2_threads(STEP), bool WITH_Q = true>
__device__ __forceinline__ void build_tile_integral(const uint8_t* __restrict__ U, uint32_t* __restrict__ T,
                                                    uint32_t* __restrict__ Q) {
    using G = TileGeoF<STEP>;
    constexpr int TW = G::TW, TH = G::TH, PW = G::PW, PH = G::PH, U8W = G::U8W;
    constexpr int NSEG = f1_nseg(PH * 256 / THREADS), SEGW = (PW + NSEG - 1) / NSEG;
    constexpr bool KEEP = SEGW <= 24;          // segment pixels kept in registers between the sweeps
    static_assert(NSEG * PH <= THREADS && (32 % NSEG) == 0, "row-pass jobs must fit one pass of the block");
    (void)Q;
    const int tid = threadIdx.x;
    const int r = tid / NSEG, sg = tid % NSEG;
    const bool act = r < PH;
    const int c0 = sg * SEGW;
    const uint8_t* row = U + r * U8W + c0;
    // sweep 1: segment totals (only the last segment can reach past PW)
    uint32_t px[KEEP ? SEGW : 1];
    uint32_t ts = 0, tq = 0;
#pragma unroll
    for (int i = 0; i < SEGW; ++i) {
        const uint32_t v = (act && c0 + i < PW) ? (uint32_t)row[i] : 0u;
        if constexpr (KEEP) px[i] = v;
        ts += v;
        tq += v * v;
    }
    uint32_t is = ts, iq = tq;                  // inclusive scan over the row's segments
#pragma unroll
    for (int d = 1; d < NSEG; d <<= 1) {
        const uint32_t a = __shfl_up_sync(0xffffffffu, is, d, NSEG);
        const uint32_t b = __shfl_up_sync(0xffffffffu, iq, d, NSEG);
        if (sg >= d) {
            is += a;
            iq += b;
        }
    }
    // sweep 2: running row prefixes of p and p^2 (exclusive segment offset + segment prefix)
    if (act) {
        uint32_t rs = is - ts, rq = iq - tq;
        uint32_t* To = T + (r + 1) * TW + 1 + c0;
        uint32_t* Qo = WITH_Q ? Q + (r + 1) * TW + 1 + c0 : nullptr;
#pragma unroll
        for (int i = 0; i < SEGW; ++i) {
            uint32_t v;
            if constexpr (KEEP)
                v = px[i];
            else
                v = c0 + i < PW ? (uint32_t)row[i] : 0u;
            rs += v;
            rq += v * v;
            if (c0 + i < PW) {
                To[i] = rs;
                if constexpr (WITH_Q) Qo[i] = rq;
            }
        }
    }
    for (int i = tid; i < TW; i += THREADS) {
        T[i] = 0u;
        if constexpr (WITH_Q) Q[i] = 0u;
    }
    for (int i = tid; i < TH; i += THREADS) {
        T[i * TW] = 0u;
        if constexpr (WITH_Q) Q[i * TW] = 0u;
    }
    __syncthreads();
    // column pass: thread per (column, plane), every row unrolled (independent loads, one add
    // chain)
    for (int j = tid; j < (WITH_Q ? 2 : 1) * PW; j += THREADS) {
        uint32_t* P = (j < PW ? T : Q) + 1 + (j < PW ? j : j - PW);
        uint32_t acc = 0;
#pragma unroll
        for (int y = 1; y < TH; ++y) {
            acc += P[y * TW];
            P[y * TW] = acc;
        }
    }
    __syncthreads();
}

// k_deep1: the deeper stages, one tile per (small) CTA and many CTAs per SM.  Each CTA claims a
// tile with stage-1 survivors, TMAs its ii plane and runs deep_phase over the survivors (in
// chunks of CP); with ~25 KB of shared memory and 4 warps per CTA, FD_K2D_CTAS tiles are in
// flight per SM, so the latency-bound stage chains of different tiles overlap.
// The deep stages of tiles claimed in order from p.deep_counter, by THREADS threads starting at
// TID0 synchronising on barrier BAR (0: the whole CTA).
template <int STEP, bool DEPTH, bool F1, int THREADS, int TID0, int BAR>
__device__ __forceinline__ void deep_tiles(const CascadeParams& p, uint8_t* smem_raw) {
    using G = TileGeoD<STEP, F1>;
    constexpr int CP = G::CP, PLANE = tile_w(STEP) * tile_h(STEP);
    uint32_t* slot = reinterpret_cast<uint32_t*>(smem_raw);
    float* pnf = reinterpret_cast<float*>(smem_raw + G::OFF_NF);
    uint16_t* ploc = reinterpret_cast<uint16_t*>(smem_raw + G::OFF_LOC);
    uint16_t* lists = reinterpret_cast<uint16_t*>(smem_raw + G::OFF_LIST);
    uint8_t* U = smem_raw + G::OFF_U8;                                       // f1: level pixels (TMA)
    __shared__ __align__(8) uint64_t mbar;
    __shared__ int s_frame[1], s_lvl[1], s_wx0[1], s_wy0[1];
    __shared__ int s_cnt[3];
    __shared__ int s_tpos, s_tile, s_off, s_n;
    const int tid = (int)threadIdx.x - TID0;
    const WinOut<STEP, DEPTH> out{p, s_frame, s_lvl, s_wx0, s_wy0};
    if (tid == 0) {
        mbar_init(&mbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    uint32_t phase = 0;
    for (;;) {
        phase_sync<BAR, THREADS>();
        if (tid == 0) {
            int tn;
            uint2 tr = make_uint2(0u, 0u);
            do {
                tn = (int)atomicAdd(p.deep_counter, 1u);
                if (tn >= p.total_tiles) break;
                tr = p.tile_rec[tn];
            } while (tr.y == 0u);
            s_tile = tn;
            if (tn < p.total_tiles) {
                const TileAt t = tile_at<STEP>(p, tn);
                s_frame[0] = p.frame_base + t.g;
                s_lvl[0] = t.k;
                s_wx0[0] = t.wx0;
                s_wy0[0] = t.wy0;
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                if (F1) {       // the tile's level pixels; its ii plane is rebuilt below
                    mbar_expect_tx(&mbar, TileGeoF<STEP>::U8W * TileGeoF<STEP>::PH);
                    tma_load_3d(U, p.tmaps + t.k, t.x, t.y, t.g, &mbar);
                } else {
                    mbar_expect_tx(&mbar, PLANE * 4);
                    tma_load_4d(slot, p.tmaps + t.k, t.x, t.y, 0, t.g, &mbar);
                }
                s_off = (int)tr.x;
                s_n = (int)tr.y;
            }
        }
        phase_sync<BAR, THREADS>();
        if (s_tile >= p.total_tiles) break;
        const int off = s_off, n = s_n;
        for (int c0 = 0; c0 < n; c0 += CP) {
            const int m = min(CP, n - c0);
            if (c0) phase_sync<BAR, THREADS>();   // previous chunk's deep phase done with the pool
            for (int e = tid; e < m; e += THREADS) {
                const uint2 v = p.surv[off + c0 + e];
                ploc[e] = (uint16_t)v.x;
                pnf[e] = __int_as_float((int)v.y);
            }
            if (tid == 0) {
                s_cnt[0] = 0;
                s_cnt[1] = 0;
                s_cnt[2] = 0;
                s_cnt[p.s0 % 3] = m;
            }
            if (c0 == 0) {
                mbar_wait(&mbar, phase);
                phase ^= 1;
                if constexpr (F1) build_tile_integral<STEP, THREADS, false>(U, slot, nullptr);
            }
            phase_sync<BAR, THREADS>();
            deep_phase<STEP, DEPTH, CP, THREADS, TID0, BAR>(p, p.s0, slot, pnf, ploc, lists, s_cnt, s_tpos, out,
                                                           reinterpret_cast<float2*>(smem_raw + G::OFF_RED));
        }
    }
}

template <int STEP, bool DEPTH, bool F1 = false>
__global__ void __launch_bounds__(K2D_THREADS, FD_K2D_CTAS) k_deep1(const __grid_constant__ CascadeParams p) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    deep_tiles<STEP, DEPTH, F1, K2D_THREADS, 0, 0>(p, smem_raw);
}


// k_f1: persistent over every (frame, level, tile) of a frame group, like k_cascade, with the
// tile's planes built in shared memory (above) instead of TMA'd from a global integral:
//   TMA box of level pixels -> tile-local ii + sqii -> variance (oracle c5) -> dense first stage
//   (run-time specialised for step 1) -> ballot compaction into the pool (over the dead sqii
//   plane) -> deep_phase (stages 1.., tail queue once few windows remain; k_tail rebuilds the
//   window's 25 x 25 ii from the same level image).
template <int STEP, bool DEPTH>
__global__ void __launch_bounds__(k2_threads(STEP), FD_F1_CTAS) k_f1(const __grid_constant__ CascadeParams p) {
    using G = TileGeoF<STEP>;
    constexpr int TW = G::TW, TX = k2_tx(STEP), TY = k2_ty(STEP), WPT = k2_wpt(STEP), CP = G::CP;
    constexpr int WARPS_X = TX / 32;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint32_t* T = reinterpret_cast<uint32_t*>(smem_raw + G::OFF_T);           // ii plane
    uint32_t* Q = reinterpret_cast<uint32_t*>(smem_raw + G::OFF_Q);           // sqii plane
    float* pnf = reinterpret_cast<float*>(smem_raw + G::OFF_NF);              // pool, over Q after stage 1
    uint16_t* ploc = reinterpret_cast<uint16_t*>(smem_raw + G::OFF_LOC);
    uint16_t* lists = reinterpret_cast<uint16_t*>(smem_raw + G::OFF_LIST);
    __shared__ __align__(8) uint64_t mbar[2];
    __shared__ int s_tile[2], s_frame[2], s_lvl[2], s_wx0[2], s_wy0[2];
    __shared__ int s_cnt[3];
    __shared__ int s_tpos, s_off;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const StageDev& st0 = p.pstages[0];
    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};
    // tid 0: claim the next tile for u8 buffer b and start its TMA
    auto claim = [&](int b) {
        const int tn = (int)atomicAdd(p.tile_counter, 1u);
        s_tile[b] = tn;
        if (tn < p.total_tiles) {
            const TileAt t = tile_at<STEP>(p, tn);
            s_frame[b] = p.frame_base + t.g;
            s_lvl[b] = t.k;
            s_wx0[b] = t.wx0;
            s_wy0[b] = t.wy0;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_expect_tx(&mbar[b], G::U8W * G::PH);
            tma_load_3d(smem_raw + b * G::UB, p.tmaps + t.k, t.x, t.y, t.g, &mbar[b]);
        }
    };
    if (tid == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        claim(0);
    }
    uint32_t phases = 0;
    for (int it = 0;; ++it) {
        const int b = it & 1;
        if (tid == 0) {
            s_cnt[0] = 0;
            s_cnt[1] = 0;
            s_cnt[2] = 0;
        }
        __syncthreads();                          // previous tile done: planes, pool, s_* of slot b^1 free
        if (s_tile[b] >= p.total_tiles) break;
        if (tid == 0) claim(b ^ 1);               // the other u8 buffer was consumed by the last build
#ifdef FD_K2_TIMING
        const long long tm0 = clock64();
#endif
        mbar_wait(&mbar[b], (phases >> b) & 1u);
        phases ^= 1u << b;
#ifdef FD_K2_TIMING
        const long long tm1 = clock64();
#endif
        build_tile_integral<STEP>(smem_raw + b * G::UB, T, Q);
#ifdef FD_K2_TIMING
        const long long tmb = clock64();
#endif
        const WinOut<STEP, DEPTH> out{p, s_frame + b, s_lvl + b, s_wx0 + b, s_wy0 + b};
        const int k = s_lvl[b];
        const int nx = __ldg(&p.lv[k].nx), ny = __ldg(&p.lv[k].ny);
        const int wx0 = s_wx0[b], wy0 = s_wy0[b];
        const int lx = lane + 32 * (warp % WARPS_X);
        const int ly0 = (warp / WARPS_X) * WPT;
        const int base = ly0 * STEP * TW + lx * STEP;
        const bool colok = wx0 + lx < nx;
        float nf[WPT], sm[WPT];
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int bo = base + i * STEP * TW;
            const uint32_t S = T[bo + WIN * TW + WIN] - T[bo + WIN] - T[bo + WIN * TW] + T[bo];
            const uint32_t q = Q[bo + WIN * TW + WIN] - Q[bo + WIN] - Q[bo + WIN * TW] + Q[bo];
            const long long v = 576LL * (long long)q - (long long)S * (long long)S;
            nf[i] = v > 0 ? __fsqrt_rn(__ll2float_rn(v)) : 1.0f;
            sm[i] = 0.0f;
        }
#ifdef FD_JIT_STAGE1
        jit_stage1(T + base, nf, sm);
#else
        if (st0.first + st0.n <= p.n_pstumps)
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, prec, st0.first, st0.n);
        else
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, grec, st0.first, st0.n);
#endif
        __syncthreads();                          // every sqii read done: the buffer becomes the pool
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int wy = wy0 + ly0 + i;
            const bool valid = colok && wy < ny;
            const bool pass = valid && (sm[i] >= st0.T);
            const int idx = (ly0 + i) * TX + lx;
            if (DEPTH && valid && !pass) out.reject(0, idx, 0, sm[i]);
            if (p.n_stages == 1) {
                if (pass) out.emit(0, idx, sm[i]);
                continue;
            }
            const unsigned m = __ballot_sync(0xffffffffu, pass);
            if (m) {
                int pos = 0;
                if (lane == 0) pos = atomicAdd(&s_cnt[1], __popc(m));
                pos = __shfl_sync(0xffffffffu, pos, 0);
                if (pass) {
                    const int at = pos + __popc(m & ((1u << lane) - 1u));
                    ploc[at] = (uint16_t)idx;
                    pnf[at] = nf[i];
                }
            }
        }
        if (tid == 0 && p.stage_counts)
            atomicAdd(p.stage_counts, (unsigned long long)min(TX, nx - wx0) * (unsigned long long)min(TY, ny - wy0));
        __syncthreads();                          // pool complete
#ifdef FD_K2_TIMING
        if (tid == 0) {
            atomicAdd(&g_k2_timing[0], 1ull);
            atomicAdd(&g_k2_timing[1], (unsigned long long)(tm1 - tm0));
            atomicAdd(&g_k2_timing[85], (unsigned long long)(tmb - tm1));
            atomicAdd(&g_k2_timing[2], (unsigned long long)(clock64() - tmb));
        }
#endif
        if (!p.surv) {
            deep_phase<STEP, DEPTH, CP>(p, 1, T, pnf, ploc, lists, s_cnt, s_tpos, out,
                                        reinterpret_cast<float2*>(smem_raw + G::OFF_RED));
            continue;
        }
        // split f1 (p.surv set): stage 1 over the pool here, one lane per window; its survivors
        // (window index, nf) go to the global list at an offset reserved for this tile, and
        // k_deep1 rebuilds the tile's ii from the same level image for the deeper stages
        const int c = s_cnt[1];
        if (tid == 0) {
            s_off = c ? (int)atomicAdd(p.surv_count, (unsigned)c) : 0;
            if (p.stage_counts && c) atomicAdd(p.stage_counts + 1, (unsigned long long)c);
        }
        __syncthreads();
        const int off = s_off;
        const StageDev& sd = p.pstages[1];
        const bool last = p.n_stages == 2;
        for (int e0 = warp * 32; e0 < c; e0 += k2_threads(STEP)) {
            const int e = e0 + lane;
            const bool act = e < c;
            int idx = 0;
            float nfw = 1.0f, sum = 0.0f;
            if (act) {
                idx = ploc[e];
                nfw = pnf[e];
                const int bo = (idx / TX) * STEP * TW + (idx % TX) * STEP;
#if FD_JIT_DEEP > 1
                sum = jit_deep(1, T + bo, nfw);
#else
                sum = sd.first + sd.n <= p.n_pstumps ? eval_stage(T, bo, nfw, prec, sd.first, sd.n, sd.mc)
                                                     : eval_stage(T, bo, nfw, grec, sd.first, sd.n, sd.mc);
#endif
            }
            const bool pass = act && (sum >= sd.T);
            if (act && !pass) out.reject(0, idx, 1, sum);
            if (last) {
                if (pass) out.emit(0, idx, sum);
                continue;
            }
            const unsigned m = __ballot_sync(0xffffffffu, pass);
            if (m) {
                int pos = 0;
                if (lane == 0) pos = atomicAdd(&s_cnt[2], __popc(m));
                pos = __shfl_sync(0xffffffffu, pos, 0);
                if (pass)
                    p.surv[off + pos + __popc(m & ((1u << lane) - 1u))] =
                        make_uint2((unsigned)idx, (unsigned)__float_as_int(nfw));
            }
        }
        __syncthreads();
        if (tid == 0) p.tile_rec[s_tile[b]] = make_uint2((unsigned)off, (unsigned)s_cnt[2]);
    }
}

}  // namespace fdk
#include "k_deepq.cuh"
namespace fdk {

#ifndef __CUDACC_RTC__
// ------------------------------------------------------------------ host launchers
// build.py compiles this file once per window step (-DFD_KC_STEP=1..4, in parallel): each object
// instantiates only its own step's kernels (StepLaunch<FD_KC_STEP>), and the step-1 object also
// holds the dispatchers over the step.  Without FD_KC_STEP every step is instantiated here.
template <int STEP, bool DEPTH>
static cudaError_t launch_stage1_t(const CascadeParams& p, cudaStream_t st) {
    static int grid = 0;
    const size_t smem = TileGeoA<STEP>::SMEM;
    cudaError_t e = cudaFuncSetAttribute(k_stage1<STEP, DEPTH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    if (!grid) {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_stage1<STEP, DEPTH>, k2_threads(STEP), smem);
        grid = sms * (per > 0 ? per : 1);
    }
    k_stage1<STEP, DEPTH><<<grid < p.total_tiles ? grid : p.total_tiles, k2_threads(STEP), smem, st>>>(p);
    return cudaGetLastError();
}


template <int STEP, bool DEPTH, bool F1>
static cudaError_t launch_deep1_t(const CascadeParams& p, cudaStream_t st) {
    static int grid = 0;
    const size_t smem = TileGeoD<STEP, F1>::SMEM;
    cudaError_t e = cudaFuncSetAttribute(k_deep1<STEP, DEPTH, F1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    if (!grid) {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_deep1<STEP, DEPTH, F1>, K2D_THREADS, smem);
        grid = sms * (per > 0 ? per : 1);
    }
    k_deep1<STEP, DEPTH, F1><<<grid < p.total_tiles ? grid : p.total_tiles, K2D_THREADS, smem, st>>>(p);
    return cudaGetLastError();
}

template <int STEP, bool DEPTH>
static cudaError_t launch_deepq_t(const CascadeParams& p, cudaStream_t st) {
    static int grid = 0;
    const size_t smem = TileGeoQ<STEP>::SMEM;
    cudaError_t e = cudaFuncSetAttribute(k_deepq<STEP, DEPTH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    if (!grid) {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_deepq<STEP, DEPTH>, DQ_THREADS, smem);
        grid = sms * (per > 0 ? per : 1);
    }
    k_deepq<STEP, DEPTH><<<grid, DQ_THREADS, smem, st>>>(p);
    return cudaGetLastError();
}


template <int STEP, bool DEPTH>
static cudaError_t launch_f1_t(const CascadeParams& p, cudaStream_t st) {
    static int grid = 0;
    const size_t smem = TileGeoF<STEP>::SMEM;
    cudaError_t e = cudaFuncSetAttribute(k_f1<STEP, DEPTH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    if (!grid) {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_f1<STEP, DEPTH>, k2_threads(STEP), smem);
        grid = sms * (per > 0 ? per : 1);
    }
    k_f1<STEP, DEPTH><<<grid < p.total_tiles ? grid : p.total_tiles, k2_threads(STEP), smem, st>>>(p);
    return cudaGetLastError();
}


template <int STEP>
struct StepLaunch {
    static cudaError_t stage1(const CascadeParams& p, bool d, cudaStream_t st) {
        return d ? launch_stage1_t<STEP, true>(p, st) : launch_stage1_t<STEP, false>(p, st);
    }
    static cudaError_t deep1(const CascadeParams& p, bool d, bool f1, cudaStream_t st) {
        if (f1) return d ? launch_deep1_t<STEP, true, true>(p, st) : launch_deep1_t<STEP, false, true>(p, st);
        return d ? launch_deep1_t<STEP, true, false>(p, st) : launch_deep1_t<STEP, false, false>(p, st);
    }
    static cudaError_t deepq(const CascadeParams& p, bool d, cudaStream_t st) {
        return d ? launch_deepq_t<STEP, true>(p, st) : launch_deepq_t<STEP, false>(p, st);
    }
    static cudaError_t f1(const CascadeParams& p, bool d, cudaStream_t st) {
        return d ? launch_f1_t<STEP, true>(p, st) : launch_f1_t<STEP, false>(p, st);
    }
};

#ifdef FD_KC_STEP
template struct StepLaunch<FD_KC_STEP>;
#endif

#if !defined(FD_KC_STEP) || FD_KC_STEP == 1
#ifdef FD_KC_STEP
extern template struct StepLaunch<2>;
extern template struct StepLaunch<3>;
extern template struct StepLaunch<4>;
#endif
#define FD_STEP_SWITCH(step, call)                   \
    switch (step) {                                   \
        case 1: return StepLaunch<1>::call;           \
        case 2: return StepLaunch<2>::call;           \
        case 3: return StepLaunch<3>::call;           \
        case 4: return StepLaunch<4>::call;           \
        default: return cudaErrorInvalidValue;        \
    }

cudaError_t launch_stage1(const CascadeParams& p, bool depth, int step, cudaStream_t st) {
    FD_STEP_SWITCH(step, stage1(p, depth, st))
}
cudaError_t launch_deep1(const CascadeParams& p, bool depth, int step, bool f1, cudaStream_t st) {
    FD_STEP_SWITCH(step, deep1(p, depth, f1, st))
}
cudaError_t launch_deepq(const CascadeParams& p, bool depth, int step, cudaStream_t st) {
    FD_STEP_SWITCH(step, deepq(p, depth, st))
}
cudaError_t launch_f1(const CascadeParams& p, bool depth, int step, cudaStream_t st) {
    FD_STEP_SWITCH(step, f1(p, depth, st))
}
#undef FD_STEP_SWITCH
#endif

#endif  // !__CUDACC_RTC__

}  // namespace fdk
