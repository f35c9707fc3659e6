// k_cascade.cu -- K2: persistent cascade evaluator over every window of every pyramid level.
//
// Paper: each integral image is cut into n x m chunks, one thread block per
// chunk, one thread per window; each block stages its chunk (2n x 2m values, eqs. 1-4) in
// shared memory, then every thread walks the stages with early exit; feature attributes sit
// in constant memory for warp-uniform broadcast.  B200 design:
//   * one persistent launch covers every (frame, level, tile) of a frame group -- replaces
//     the paper's one-kernel-per-scale streams;
//   * a tile of TX x TY windows needs a (TX+24) x (TY+24) block of ii and sqii: one 4-D TMA
//     (cp.async.bulk.tensor) per tile, double buffered with mbarriers, prefetching the next
//     tile while the current one is evaluated;
//   * stage 1 (94.5% of windows stop there) is evaluated densely: each thread
//     owns 8 windows of a column, stump records are warp-uniform loads, and each Haar
//     feature is pre-compiled on the host into its distinct integral-image corners with
//     integer coefficients (sum_r wt_r*R_r == sum_c coef_c*ii_c exactly, mod 2^32);
//   * survivors are compacted with warp ballots into a shared-memory queue after every stage
//     so deeper stages run on full warps (the divergence problem of P:L1228-1258);
//   * fp32 arithmetic matches the oracle bit for bit: __fmul_rn/__fadd_rn (no FMA
//     contraction), __int2float_rn, __ll2float_rn, IEEE __fsqrt_rn.
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

// One stage for one window: sum_j leaf_j in stump order (oracle c7/c8).
template <int STEP>
__device__ __forceinline__ float eval_stage(const uint32_t* __restrict__ T, int b, float nf, const uint4* __restrict__ rec,
                                            int n) {
    float sum = 0.0f;
    for (int j = 0; j < n; ++j) {
        const uint4 h = __ldg(rec + 4 * j);
        const uint4 c0 = __ldg(rec + 4 * j + 1), c1 = __ldg(rec + 4 * j + 2), c2 = __ldg(rec + 4 * j + 3);
        const int nc = (int)h.x;
        uint32_t f = 0;
#pragma unroll
        for (int c = 0; c < MAX_CORNERS; ++c) {
            if (c < nc) {
                const int w = corner_word(c0, c1, c2, c);
                f += (uint32_t)(w >> 16) * T[b + (w & 0xffff)];
            }
        }
        const float t = __fmul_rn(__int_as_float((int)h.y), nf);
        const float leaf = (__int2float_rn((int)f) < t) ? __int_as_float((int)h.z) : __int_as_float((int)h.w);
        sum = __fadd_rn(sum, leaf);
    }
    return sum;
}

// below this many surviving windows a deep stage runs warp-per-window / lane-per-stump
constexpr int LANE_MODE_MIN = 64;

__device__ __forceinline__ int find_level_tile(const PlanDev& p, int r) {
    int k = 0;
    while (k + 1 < p.n_levels && p.lv[k + 1].tile0 <= r) ++k;
    return k;
}

template <int STEP>
struct TileGeo {
    static constexpr int TX = k2_tx(STEP);
    static constexpr int TY = k2_ty(STEP);
    static constexpr int WPT = k2_wpt(STEP);
    static constexpr int WARPS_X = TX / 32;
    static constexpr int TW = tile_w(STEP);
    static constexpr int TH = tile_h(STEP);
    static constexpr int PLANE = TW * TH;          // u32 per plane
    static constexpr int BOX = 2 * PLANE;          // ii + sqii (one TMA box)
    static constexpr int BUF = (BOX + 255) & ~255; // buffer stride: keeps every TMA destination 1 KB aligned
    static constexpr int NW = TX * TY;             // windows per tile
    static constexpr size_t SMEM = (size_t)2 * BUF * 4 + (size_t)NW * 4 * 2 + (size_t)NW * 2 * 2;
};

template <int STEP, bool DEPTH>
__global__ void __launch_bounds__(K2_THREADS, 2) k_cascade(const __grid_constant__ CascadeParams p) {
    using G = TileGeo<STEP>;
    constexpr int TW = G::TW, TX = G::TX, TY = G::TY, WPT = G::WPT;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint32_t* tiles = reinterpret_cast<uint32_t*>(smem_raw);               // [2][2][TH][TW]
    float* nfs = reinterpret_cast<float*>(tiles + 2 * G::BUF);              // [NW] per-window nf
    float* sums = nfs + G::NW;                                              // [NW] last stage sum
    uint16_t* lists = reinterpret_cast<uint16_t*>(sums + G::NW);            // [2][NW]
    __shared__ __align__(8) uint64_t mbar[2];
    __shared__ int s_tile[2];
    __shared__ int s_cnt[3];

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int N = p.n_stages;
    const StageDev st0 = p.stages[0];

    if (tid == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        const int t0 = (int)atomicAdd(p.tile_counter, 1u);
        s_tile[0] = t0;
        if (t0 < p.total_tiles) {
            const int g = t0 / p.plan.tiles_per_frame, r = t0 % p.plan.tiles_per_frame;
            const int k = find_level_tile(p.plan, r);
            const LevelDev& L = p.plan.lv[k];
            const int tl = r - L.tile0;
            mbar_expect_tx(&mbar[0], G::BOX * 4);
            tma_load_4d(tiles, &p.tmap[k], (tl % L.tiles_x) * TX * STEP, (tl / L.tiles_x) * TY * STEP, 0, g, &mbar[0]);
        }
    }
    uint32_t phase0 = 0, phase1 = 0;

    for (int it = 0;; ++it) {
        const int buf = it & 1;
        __syncthreads();                      // previous tile fully consumed (buf^1 free, counters free)
        if (tid == 0) {
            s_cnt[0] = 0;
            s_cnt[1] = 0;
            s_cnt[2] = 0;
            const int tn = (int)atomicAdd(p.tile_counter, 1u);
            s_tile[buf ^ 1] = tn;
            if (tn < p.total_tiles) {
                const int g = tn / p.plan.tiles_per_frame, r = tn % p.plan.tiles_per_frame;
                const int k = find_level_tile(p.plan, r);
                const LevelDev& L = p.plan.lv[k];
                const int tl = r - L.tile0;
                mbar_expect_tx(&mbar[buf ^ 1], G::BOX * 4);
                tma_load_4d(tiles + (buf ^ 1) * G::BUF, &p.tmap[k], (tl % L.tiles_x) * TX * STEP,
                            (tl / L.tiles_x) * TY * STEP, 0, g, &mbar[buf ^ 1]);
            }
        }
        __syncthreads();
        const int t = s_tile[buf];
        if (t >= p.total_tiles) break;
        const int g = t / p.plan.tiles_per_frame, r = t % p.plan.tiles_per_frame;
        const int k = find_level_tile(p.plan, r);
        const LevelDev& L = p.plan.lv[k];
        const int tl = r - L.tile0;
        const int wx0 = (tl % L.tiles_x) * TX, wy0 = (tl / L.tiles_x) * TY;
        const int frame = p.frame_base + g;
        if (buf == 0) {
            mbar_wait(&mbar[0], phase0);
            phase0 ^= 1;
        } else {
            mbar_wait(&mbar[1], phase1);
            phase1 ^= 1;
        }
        const uint32_t* T = tiles + buf * G::BUF;      // ii plane
        const uint32_t* Q = T + G::PLANE;              // sqii plane (mod 2^32)

        // ---------------- stage 1, dense: 8 windows per thread down a column
        const int lx = lane + 32 * (warp % G::WARPS_X);
        const int ly0 = (warp / G::WARPS_X) * WPT;
        const int base = ly0 * STEP * TW + lx * STEP;
        const bool colok = wx0 + lx < L.nx;
        float nf[WPT], sm[WPT];
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int b = base + i * STEP * TW;
            const uint32_t S = T[b + WIN * TW + WIN] - T[b + WIN] - T[b + WIN * TW] + T[b];
            const uint32_t q = Q[b + WIN * TW + WIN] - Q[b + WIN] - Q[b + WIN * TW] + Q[b];
            const long long v = 576LL * (long long)q - (long long)S * (long long)S;
            nf[i] = v > 0 ? __fsqrt_rn(__ll2float_rn(v)) : 1.0f;
            nfs[(ly0 + i) * TX + lx] = nf[i];
            sm[i] = 0.0f;
        }
        {
            const uint4* rec = p.stumps + 4 * st0.first;
            for (int j = 0; j < st0.n; ++j) {
                const uint4 h = __ldg(rec + 4 * j);
                const uint4 c0 = __ldg(rec + 4 * j + 1), c1 = __ldg(rec + 4 * j + 2), c2 = __ldg(rec + 4 * j + 3);
                const int nc = (int)h.x;
                uint32_t f[WPT];
#pragma unroll
                for (int i = 0; i < WPT; ++i) f[i] = 0;
#pragma unroll
                for (int c = 0; c < MAX_CORNERS; ++c) {
                    if (c < nc) {
                        const int w = corner_word(c0, c1, c2, c);
                        const uint32_t coef = (uint32_t)(w >> 16);
                        const uint32_t* src = T + base + (w & 0xffff);
#pragma unroll
                        for (int i = 0; i < WPT; ++i) f[i] += coef * src[i * STEP * TW];
                    }
                }
                const float th = __int_as_float((int)h.y), lf = __int_as_float((int)h.z), rt = __int_as_float((int)h.w);
#pragma unroll
                for (int i = 0; i < WPT; ++i) {
                    const float tt = __fmul_rn(th, nf[i]);
                    sm[i] = __fadd_rn(sm[i], (__int2float_rn((int)f[i]) < tt) ? lf : rt);
                }
            }
        }
        // compaction of stage-1 survivors into lists[1] (count s_cnt[1])
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int wy = wy0 + ly0 + i;
            const bool valid = colok && wy < L.ny;
            const bool pass = valid && (sm[i] >= st0.T);
            const int idx = (ly0 + i) * TX + lx;
            if (DEPTH && valid && !pass) {
                const long long o = (long long)frame * p.plan.win_per_frame + L.win0 + (long long)wy * L.nx + (wx0 + lx);
                p.depth[o] = 0;
                p.score[o] = sm[i];
            }
            const unsigned m = __ballot_sync(0xffffffffu, pass);
            if (m) {
                int pos = 0;
                if (lane == 0) pos = atomicAdd(&s_cnt[1], __popc(m));
                pos = __shfl_sync(0xffffffffu, pos, 0);
                if (pass) {
                    const int at = pos + __popc(m & ((1u << lane) - 1u));
                    lists[G::NW + at] = (uint16_t)idx;
                    sums[idx] = sm[i];
                }
            }
        }
        if (tid == 0 && p.stage_counts) {
            const unsigned long long nv =
                (unsigned long long)min(TX, L.nx - wx0) * (unsigned long long)min(TY, L.ny - wy0);
            atomicAdd(p.stage_counts, nv);
        }
        __syncthreads();

        // ---------------- deeper stages over the compacted queue
        int s = 1;
        for (; s < N; ++s) {
            const int n = s_cnt[s % 3];
            if (tid == 0 && p.stage_counts && n) atomicAdd(p.stage_counts + s, (unsigned long long)n);
            if (n == 0) break;
            if (tid == 0) s_cnt[(s + 2) % 3] = 0;
            const StageDev sd = p.stages[s];
            const uint16_t* lin = lists + (s & 1) * G::NW;
            uint16_t* lout = lists + ((s + 1) & 1) * G::NW;
            const uint4* rec = p.stumps + 4 * sd.first;
            if (n < LANE_MODE_MIN) {
                // few survivors: one warp per window, one lane per stump (params and corners
                // fetched in parallel), then the leaves are added in stump order (exact fp32
                // sequence of the definition) by every lane redundantly via shuffles.
                for (int e = warp; e < n; e += K2_THREADS / 32) {
                    const int idx = lin[e];
                    const int wlx = idx % TX, wly = idx / TX;
                    const int b = wly * STEP * TW + wlx * STEP;
                    const float nfw = nfs[idx];
                    float sum = 0.0f;
                    for (int c0 = 0; c0 < sd.n; c0 += 32) {
                        const int j = c0 + lane;
                        float leaf = 0.0f;
                        if (j < sd.n) leaf = eval_stage<STEP>(T, b, nfw, rec + 4 * j, 1);
                        const int m = min(32, sd.n - c0);
                        for (int t = 0; t < m; ++t) sum = __fadd_rn(sum, __shfl_sync(0xffffffffu, leaf, t));
                    }
                    if (lane == 0) {
                        if (sum >= sd.T) {
                            lout[atomicAdd(&s_cnt[(s + 1) % 3], 1)] = (uint16_t)idx;
                            sums[idx] = sum;
                        } else if (DEPTH) {
                            const long long o = (long long)frame * p.plan.win_per_frame + L.win0 +
                                                (long long)(wy0 + wly) * L.nx + (wx0 + wlx);
                            p.depth[o] = (uint8_t)(s < 255 ? s : 255);
                            p.score[o] = sum;
                        }
                    }
                }
                __syncthreads();
                continue;
            }
            for (int e0 = warp * 32; e0 < n; e0 += K2_THREADS) {
                const int e = e0 + lane;
                const bool act = e < n;
                int idx = 0;
                float sum = 0.0f;
                if (act) {
                    idx = lin[e];
                    const int wlx = idx % TX, wly = idx / TX;
                    sum = eval_stage<STEP>(T, wly * STEP * TW + wlx * STEP, nfs[idx], rec, sd.n);
                }
                const bool pass = act && (sum >= sd.T);
                if (DEPTH && act && !pass) {
                    const int wlx = idx % TX, wly = idx / TX;
                    const long long o = (long long)frame * p.plan.win_per_frame + L.win0 +
                                        (long long)(wy0 + wly) * L.nx + (wx0 + wlx);
                    p.depth[o] = (uint8_t)(s < 255 ? s : 255);
                    p.score[o] = sum;
                }
                const unsigned m = __ballot_sync(0xffffffffu, pass);
                if (m) {
                    int pos = 0;
                    if (lane == 0) pos = atomicAdd(&s_cnt[(s + 1) % 3], __popc(m));
                    pos = __shfl_sync(0xffffffffu, pos, 0);
                    if (pass) {
                        lout[pos + __popc(m & ((1u << lane) - 1u))] = (uint16_t)idx;
                        sums[idx] = sum;
                    }
                }
            }
            __syncthreads();
        }
        if (s == N) {                               // accepted windows: depth N
            const int nacc = s_cnt[N % 3];
            if (tid == 0 && p.stage_counts && nacc) atomicAdd(p.stage_counts + N, (unsigned long long)nacc);
            const uint16_t* lacc = lists + (N & 1) * G::NW;
            for (int e0 = warp * 32; e0 < nacc; e0 += K2_THREADS) {
                const int e = e0 + lane;
                const bool act = e < nacc;
                int idx = act ? lacc[e] : 0;
                const int wlx = idx % TX, wly = idx / TX;
                if (DEPTH) {
                    if (act) {
                        const long long o = (long long)frame * p.plan.win_per_frame + L.win0 +
                                            (long long)(wy0 + wly) * L.nx + (wx0 + wlx);
                        p.depth[o] = (uint8_t)(N < 255 ? N : 255);
                        p.score[o] = sums[idx];
                    }
                } else {
                    const unsigned m = __ballot_sync(0xffffffffu, act);
                    unsigned long long pos = 0;
                    if (lane == 0) pos = atomicAdd(p.det_count, (unsigned long long)__popc(m));
                    pos = __shfl_sync(0xffffffffu, pos, 0);
                    if (act) {
                        const unsigned long long at = pos + __popc(m & ((1u << lane) - 1u));
                        if ((long long)at < p.det_cap) {
                            p.det_keys[at] = det_key(frame, k, (wy0 + wly) * STEP, (wx0 + wlx) * STEP);
                            p.det_scores[at] = sums[idx];
                        }
                    }
                }
            }
        }
    }
}

template <int STEP, bool DEPTH>
static cudaError_t launch_one(const CascadeParams& p, int grid, cudaStream_t st) {
    const size_t smem = TileGeo<STEP>::SMEM;
    cudaError_t e = cudaFuncSetAttribute(k_cascade<STEP, DEPTH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_cascade<STEP, DEPTH><<<grid, K2_THREADS, smem, st>>>(p);
    return cudaGetLastError();
}

template <int STEP, bool DEPTH>
static int grid_one() {
    const size_t smem = TileGeo<STEP>::SMEM;
    cudaFuncSetAttribute(k_cascade<STEP, DEPTH>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_cascade<STEP, DEPTH>, K2_THREADS, smem);
    return sms * (per > 0 ? per : 1);
}

size_t cascade_smem(int step) {
    switch (step) {
        case 1: return TileGeo<1>::SMEM;
        case 2: return TileGeo<2>::SMEM;
        case 3: return TileGeo<3>::SMEM;
        default: return TileGeo<4>::SMEM;
    }
}

int cascade_grid(bool depth, int step) {
    switch (step) {
        case 1: return depth ? grid_one<1, true>() : grid_one<1, false>();
        case 2: return depth ? grid_one<2, true>() : grid_one<2, false>();
        case 3: return depth ? grid_one<3, true>() : grid_one<3, false>();
        default: return depth ? grid_one<4, true>() : grid_one<4, false>();
    }
}

cudaError_t launch_cascade(const CascadeParams& p, bool depth, int step, int grid, cudaStream_t st) {
    switch (step) {
        case 1: return depth ? launch_one<1, true>(p, grid, st) : launch_one<1, false>(p, grid, st);
        case 2: return depth ? launch_one<2, true>(p, grid, st) : launch_one<2, false>(p, grid, st);
        case 3: return depth ? launch_one<3, true>(p, grid, st) : launch_one<3, false>(p, grid, st);
        case 4: return depth ? launch_one<4, true>(p, grid, st) : launch_one<4, false>(p, grid, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace fdk
