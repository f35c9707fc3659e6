// k_tail.cu -- K2, second kernel: the deep stages of the few windows per tile that survive the
// early stages (oracle c7/c8; P:L451-457 sequential stages with early rejection).
//
// Inside k_cascade a tile's windows are evaluated stage-synchronously: dense first stage,
// then ballot-compacted deeper stages.  Once only a handful of windows are left (c3: ~5 of
// 2048 after three or four stages, P:L1311-1325 rejection profile) the tile would wait for its
// deepest window, a serial chain of up to ~1400 stumps.  k_cascade instead appends those
// windows to a global queue and moves on to its next tile; this kernel finishes them, one warp
// per window, with no block-level synchronisation at all:
//   * the window's 25 x 25 ii region is staged in the warp's shared memory once: 25 coalesced
//     row loads of plane 0 of the group workspace, or -- on the f1 path, where no global integral
//     exists -- a window-local integral built from the window's 24 x 24 level pixels;
//   * lane j evaluates stump c0 + j of the current stage from SoA tail records (word w of
//     stump j at trec[w * ns + j]: coalesced 128-B loads) whose corner offsets address the
//     staged region directly;
//   * the stage decision comes from a warp tree sum certified against its rounding-error bound
//     (k_common.cuh certify): provably the decision of the definition's sequential fp32 sum.
//     The sequential sum itself (leaves added in stump order: independent shuffles, serial
//     adds) is computed only for near ties and for the scores that are outputs (the last stage
//     of an accepted window, the rejecting stage in depth mode).
#include "k_common.cuh"

namespace fdk {

constexpr int TAIL_THREADS = 256;
template <int V>
struct IntC {
    static constexpr int value = V;
};
constexpr int TAIL_REGION = ((WIN + 1) * TAIL_RP + 31) & ~31;   // words per warp

// Dynamic shared memory: the SoA records of stumps [j0, j0 + nsm) (the early deep stages, where
// most tail windows are; word w of stump j at srec[w * nsm + j - j0]), then one 25 x 25 region per
// warp.  Stages outside that range read the records from global memory.
size_t tail_smem(int nsm) { return ((size_t)TAIL_REC_WORDS * nsm + (size_t)(TAIL_THREADS / 32) * TAIL_REGION) * 4; }

template <bool DEPTH>
__global__ void __launch_bounds__(TAIL_THREADS, 4) k_tail(const __grid_constant__ TailParams p) {
    extern __shared__ uint32_t tsm[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t* srec = tsm;
    uint32_t* R = tsm + TAIL_REC_WORDS * p.nsm + warp * TAIL_REGION;
    for (int i = threadIdx.x; i < TAIL_REC_WORDS * p.nsm; i += TAIL_THREADS) {
        const int w = i / p.nsm, j = i - w * p.nsm;
        srec[i] = __ldg(p.trec + (size_t)w * p.ns + p.j0 + j);
    }
    __syncthreads();
    const unsigned cnt = *p.count;
    const int n = (int)(cnt < (unsigned)p.cap ? cnt : (unsigned)p.cap);
    const int N = p.n_stages;
    for (int e = blockIdx.x * (TAIL_THREADS / 32) + warp; e < n; e += gridDim.x * (TAIL_THREADS / 32)) {
        const uint4 q = __ldg(p.q + e);
        const int g = (int)q.w, k = (int)((q.x >> 8) & 255), s = (int)(q.x & 255);
        const int wyi = (int)(q.y >> 16), wxi = (int)(q.y & 0xffffu);
        const float nf = __int_as_float((int)q.z);
        const LevelDev L = p.lv[k];
        __syncwarp();                         // previous window's region reads done
        if (p.lvl8) {
            // f1: no global integral exists; the window's 25 x 25 ii is built from its 24 x 24
            // level pixels (a window-local integral: rectangle sums are origin-independent, R4).
            // Lane r < 24 scans pixel row r into R[r + 1][1..24]; then lane c adds down column c.
            const uint8_t* src = p.lvl8 + L.u8_off + ((long long)g * L.H + (long long)wyi * p.step) * L.PB +
                                 (long long)wxi * p.step;
            if (lane < WIN) {
                uint8_t px[WIN];
#pragma unroll
                for (int c = 0; c < WIN; ++c) px[c] = __ldg(src + (long long)lane * L.PB + c);
                uint32_t acc = 0;
                R[(lane + 1) * TAIL_RP] = 0u;
#pragma unroll
                for (int c = 0; c < WIN; ++c) {
                    acc += px[c];
                    R[(lane + 1) * TAIL_RP + c + 1] = acc;
                }
            }
            if (lane <= WIN) R[lane] = 0u;
            __syncwarp();
            if (lane < WIN) {
                uint32_t acc = 0;
#pragma unroll
                for (int r = 1; r <= WIN; ++r) {
                    acc += R[r * TAIL_RP + lane + 1];
                    R[r * TAIL_RP + lane + 1] = acc;
                }
            }
        } else {
            const uint32_t* src = p.ws + L.ws_off + (long long)g * 2 * (L.H + 1) * L.P +
                                  (long long)(wyi * p.step) * L.P + wxi * p.step;
            if (lane <= WIN) {       // 25 independent row loads in flight, then 25 stores
                uint32_t v[WIN + 1];
#pragma unroll
                for (int r = 0; r <= WIN; ++r) v[r] = __ldg(src + (long long)r * L.P + lane);
#pragma unroll
                for (int r = 0; r <= WIN; ++r) R[r * TAIL_RP + lane] = v[r];
            }
        }
        __syncwarp();
        // leaf of stump c0 + lane of stage sd (0 beyond the stage); MC >= the stage's largest
        // corner count (unused corner slots are offset 0, coefficient 0), so the corner loads do
        // not wait for the stump's own count
        // (the shared-memory and global record paths are separate so each compiles to its own
        // address space: 32-bit LDS, or LDG through the read-only path)
        auto leaf_rec = [&](const uint32_t* t, int ws, auto mc_tag) -> float {
            constexpr int MC = decltype(mc_tag)::value;
            uint32_t f = 0;
#pragma unroll
            for (int c = 0; c < MC; ++c) {
                const uint32_t w = t[(4 + c) * ws];
                f += (uint32_t)((int)w >> 16) * R[w & 0xffffu];
            }
            const float tt = __fmul_rn(__int_as_float((int)t[ws]), nf);
            return (__int2float_rn((int)f) < tt) ? __int_as_float((int)t[2 * ws]) : __int_as_float((int)t[3 * ws]);
        };
        auto leaf_mc = [&](const StageDev& sd, int c0, auto mc_tag) -> float {
            constexpr int MC = decltype(mc_tag)::value;
            if (c0 + lane >= sd.n) return 0.0f;
            if (sd.first >= p.j0 && sd.first + sd.n <= p.j0 + p.nsm)     // stage-uniform
                return leaf_rec(srec + (sd.first - p.j0 + c0 + lane), p.nsm, IntC<MC>{});
            const uint32_t* __restrict__ g = p.trec + sd.first + c0 + lane;
            uint32_t f = 0;
#pragma unroll
            for (int c = 0; c < MC; ++c) {
                const uint32_t w = __ldg(g + (size_t)(4 + c) * p.ns);
                f += (uint32_t)((int)w >> 16) * R[w & 0xffffu];
            }
            const float tt = __fmul_rn(__int_as_float((int)__ldg(g + p.ns)), nf);
            return (__int2float_rn((int)f) < tt) ? __int_as_float((int)__ldg(g + 2 * (size_t)p.ns))
                                                 : __int_as_float((int)__ldg(g + 3 * (size_t)p.ns));
        };
        auto leaf_of = [&](const StageDev& sd, int c0) -> float {
            if (sd.mc <= 6) return leaf_mc(sd, c0, IntC<6>{});
            if (sd.mc <= 8) return leaf_mc(sd, c0, IntC<8>{});
            if (sd.mc <= 9) return leaf_mc(sd, c0, IntC<9>{});
            return leaf_mc(sd, c0, IntC<MAX_CORNERS>{});
        };
        int s2 = s;
        float sum = 0.0f;
        for (; s2 < N; ++s2) {
            const StageDev sd = p.stages[s2];
            if (s2 > s && lane == 0 && p.stage_counts) atomicAdd(p.stage_counts + s2, 1ull);
            // tree sum over the warp + certified decision (k_common.cuh certify)
            float acc = 0.0f, aacc = 0.0f;
            for (int c0 = 0; c0 < sd.n; c0 += 32) {
                const float l = leaf_of(sd, c0);
                acc = __fadd_rn(acc, l);
                aacc = __fadd_rn(aacc, fabsf(l));
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, o));
                aacc = __fadd_rn(aacc, __shfl_xor_sync(0xffffffffu, aacc, o));
            }
            int dec = certify(acc, aacc, sd.n, (sd.n + 31) / 32 - 1 + 5, sd.T);
            sum = acc;
            if (dec < 0 || (dec == 1 && s2 == N - 1) || (DEPTH && dec == 0)) {
                // the definition's sequence: leaves added in stump order (independent shuffles,
                // serial adds)
                sum = 0.0f;
                for (int c0 = 0; c0 < sd.n; c0 += 32) {
                    const float leaf = leaf_of(sd, c0);
                    const int m = min(32, sd.n - c0);
#pragma unroll
                    for (int t2 = 0; t2 < 32; ++t2) {
                        const float v = __shfl_sync(0xffffffffu, leaf, t2);
                        if (t2 < m) sum = __fadd_rn(sum, v);
                    }
                }
                dec = sum >= sd.T ? 1 : 0;
            }
            if (dec == 0) break;
        }
        if (lane == 0) {
            const int frame = p.frame_base + g;
            if (DEPTH) {
                const long long o = (long long)frame * p.win_per_frame + L.win0 + (long long)wyi * L.nx + wxi;
                p.depth[o] = (uint8_t)(s2 < 255 ? s2 : 255);
                p.score[o] = sum;
            }
            if (s2 == N) {
                if (p.stage_counts) atomicAdd(p.stage_counts + N, 1ull);
                if (!DEPTH) {
                    const unsigned long long at = atomicAdd(p.det_count, 1ull);
                    if ((long long)at < p.det_cap) {
                        p.det_keys[at] = det_key(frame, k, wyi * p.step, wxi * p.step);
                        p.det_scores[at] = sum;
                    }
                }
            }
        }
    }
}

cudaError_t launch_tail(const TailParams& p, bool depth, cudaStream_t st) {
    const size_t smem = tail_smem(p.nsm);
    cudaError_t e = cudaFuncSetAttribute(depth ? k_tail<true> : k_tail<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return e;
    int dev = 0, sms = 148, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, depth ? k_tail<true> : k_tail<false>, TAIL_THREADS, smem);
    const int grid = sms * (per > 0 ? per : 1);
    if (depth)
        k_tail<true><<<grid, TAIL_THREADS, smem, st>>>(p);
    else
        k_tail<false><<<grid, TAIL_THREADS, smem, st>>>(p);
    return cudaGetLastError();
}

}  // namespace fdk
