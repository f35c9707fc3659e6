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

constexpr int LC = 8;                        // leaves parked per lane before the ordered sum (group mode)

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
    static constexpr int THREADS = k2_threads(STEP);
    static constexpr size_t LEAVES = (size_t)THREADS * LC;   // floats
    static constexpr size_t smem(int nst) {
        return (size_t)nst * BUF * 4 + (size_t)NW * 4 * 2 + LEAVES * 4 + (size_t)NW * 2 * 2;
    }
};

// NST = TMA stages: 2 = double-buffered tiles (prefetch the next tile during evaluation),
// 1 = single buffer with one more resident CTA per SM.
template <int STEP, bool DEPTH, int NST>
__global__ void __launch_bounds__(k2_threads(STEP), k2_threads(STEP) == 128 ? 5 : (NST == 1 ? 3 : 2)) k_cascade(const __grid_constant__ CascadeParams p) {
    using G = TileGeo<STEP>;
    constexpr int TW = G::TW, TX = G::TX, TY = G::TY, WPT = G::WPT;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint32_t* tiles = reinterpret_cast<uint32_t*>(smem_raw);               // [NST][2][TH][TW]
    float* nfs = reinterpret_cast<float*>(tiles + NST * G::BUF);            // [NW] per-window nf
    float* sums = nfs + G::NW;                                              // [NW] last stage sum
    float* leaves = sums + G::NW;                                           // [8 warps][LC][32]
    uint16_t* lists = reinterpret_cast<uint16_t*>(leaves + G::LEAVES);      // [2][NW]
    __shared__ __align__(8) uint64_t mbar[2];
    __shared__ int s_tile[2], s_lvl[2], s_tl[2];
    __shared__ int s_cnt[3];

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int N = p.n_stages;
    const StageDev& st0 = p.pstages[0];     // parameter bank: warp-uniform (n_pstages >= 1)
    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};

    // thread 0: claim a tile from the work counter, decode it and start its TMA into buffer b
    auto fetch = [&](int b) {
        const int tn = (int)atomicAdd(p.tile_counter, 1u);
        s_tile[b] = tn;
        if (tn < p.total_tiles) {
            const int g = tn / p.tiles_per_frame, r = tn % p.tiles_per_frame;
            int k = 0;
            while (k + 1 < p.n_levels && __ldg(&p.lv[k + 1].tile0) <= r) ++k;
            const int tl = r - __ldg(&p.lv[k].tile0);
            const int tx = __ldg(&p.lv[k].tiles_x);
            s_lvl[b] = k;
            s_tl[b] = tl;
            mbar_expect_tx(&mbar[b], G::BOX * 4);
            tma_load_4d(tiles + b * G::BUF, p.tmaps + k, (tl % tx) * TX * STEP, (tl / tx) * TY * STEP, 0, g, &mbar[b]);
        }
    };
    if (tid == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        if (NST == 2) fetch(0);
    }
    uint32_t phase0 = 0, phase1 = 0;

    for (int it = 0;; ++it) {
        const int buf = NST == 2 ? (it & 1) : 0;
        __syncthreads();                      // previous tile fully consumed (buffers and counters free)
        if (tid == 0) {
            s_cnt[0] = 0;
            s_cnt[1] = 0;
            s_cnt[2] = 0;
            fetch(NST == 2 ? (buf ^ 1) : 0);  // double buffer: prefetch the next tile; single: this one
        }
        __syncthreads();
        const int t = s_tile[buf];
        if (t >= p.total_tiles) break;
        const int g = t / p.tiles_per_frame;
        const int k = s_lvl[buf];
        const LevelDev L = p.lv[k];
        const int tl = s_tl[buf];
        const int wx0 = (tl % L.tiles_x) * TX, wy0 = (tl / L.tiles_x) * TY;
        const int frame = p.frame_base + g;
#ifdef FD_K2_TIMING
        const long long tm0 = clock64();
#endif
        if (buf == 0) {
            mbar_wait(&mbar[0], phase0);
            phase0 ^= 1;
        } else {
            mbar_wait(&mbar[1], phase1);
            phase1 ^= 1;
        }
#ifdef FD_K2_TIMING
        const long long tm1 = clock64();
#endif
        const uint32_t* T = tiles + buf * G::BUF;      // ii plane
        const uint32_t* Q = T + G::PLANE;              // sqii plane (mod 2^32)

        // ---------------- stage 1, dense: WPT windows per thread down a column
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
#ifdef FD_JIT_STAGE1
        // run-time specialised first stage (fd_jit.cpp): corner offsets, coefficients and
        // thresholds are immediates and each (column, row) value is loaded once per thread
        jit_stage1(T + base, nf, sm);
#else
        if (st0.first + st0.n <= p.n_pstumps)
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, prec, st0.first, st0.n);
        else
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, grec, st0.first, st0.n);
#endif

        // compaction of stage-1 survivors into lists[1] (count s_cnt[1])
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int wy = wy0 + ly0 + i;
            const bool valid = colok && wy < L.ny;
            const bool pass = valid && (sm[i] >= st0.T);
            const int idx = (ly0 + i) * TX + lx;
            if (DEPTH && valid && !pass) {
                const long long o = (long long)frame * p.win_per_frame + L.win0 + (long long)wy * L.nx + (wx0 + lx);
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

#ifdef FD_K2_TIMING
        const long long tm2 = clock64();
#endif
        // ---------------- deeper stages over the compacted queue
        int s = 1;
        // one deep stage; sd is a parameter-bank (uniform) or global stage descriptor
        auto deep_stage = [&](const StageDev& sd, int n) {
            const uint16_t* lin = lists + (s & 1) * G::NW;
            uint16_t* lout = lists + ((s + 1) & 1) * G::NW;
            // stages [1, FD_JIT_DEEP) of the run-time specialised kernel: immediate-offset code,
            // always one lane per window
            const bool jit_s = FD_JIT_DEEP > 0 && s < FD_JIT_DEEP;
            if (!jit_s && n < p.lane_min) {
                // fewer windows than half the block: GL = 2^lg lanes per window (the largest
                // power of two with n*GL <= THREADS, so one pass covers every window and
                // all warps work); the group's lanes evaluate different stumps, the leader adds
                // the leaves in stump order (the exact fp32 sequence of the definition).
                int lg = 1;
                while (lg < 5 && (n << (lg + 1)) <= G::THREADS) ++lg;
                const int e = tid >> lg;
                const bool act = e < n;
                const int idx = act ? lin[e] : 0;
                const int wlx = idx % TX, wly = idx / TX;
                const int b = wly * STEP * TW + wlx * STEP;
                const float nfw = act ? nfs[idx] : 1.0f;
                const float sum = group_stage<LC>(T, b, nfw, grec, sd.first, sd.n, sd.mc, lg, act,
                                                  leaves + warp * 32 * LC, lane);
                if (act && (lane & ((1 << lg) - 1)) == 0) {
                    if (sum >= sd.T) {
                        lout[atomicAdd(&s_cnt[(s + 1) % 3], 1)] = (uint16_t)idx;
                        sums[idx] = sum;
                    } else if (DEPTH) {
                        const long long o = (long long)frame * p.win_per_frame + L.win0 +
                                            (long long)(wy0 + wly) * L.nx + (wx0 + wlx);
                        p.depth[o] = (uint8_t)(s < 255 ? s : 255);
                        p.score[o] = sum;
                    }
                }
                return;
            }
            const bool in_param = sd.first + sd.n <= p.n_pstumps;
            for (int e0 = warp * 32; e0 < n; e0 += G::THREADS) {
                const int e = e0 + lane;
                const bool act = e < n;
                int idx = 0;
                float sum = 0.0f;
                if (act) {
                    idx = lin[e];
                    const int wlx = idx % TX, wly = idx / TX;
                    const int b = wly * STEP * TW + wlx * STEP;
#if FD_JIT_DEEP > 0
                    if (jit_s)
                        sum = jit_deep(s, T + b, nfs[idx]);
                    else
#endif
                        sum = in_param ? eval_stage(T, b, nfs[idx], prec, sd.first, sd.n, sd.mc)
                                       : eval_stage(T, b, nfs[idx], grec, sd.first, sd.n, sd.mc);
                }
                const bool pass = act && (sum >= sd.T);
                if (DEPTH && act && !pass) {
                    const int wlx = idx % TX, wly = idx / TX;
                    const long long o = (long long)frame * p.win_per_frame + L.win0 +
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
        };
        bool tail_done = false;
        for (; s < N; ++s) {
#ifdef FD_K2_TIMING
            const long long ts0 = clock64();
#endif
            const int n = s_cnt[s % 3];
            if (tid == 0 && p.stage_counts && n) atomicAdd(p.stage_counts + s, (unsigned long long)n);
            if (n == 0) break;
            if (n <= G::THREADS / 32 && !(FD_JIT_DEEP > 0 && s < FD_JIT_DEEP)) {
                // tail: at most one window per warp left -- each warp walks its window through
                // all remaining stages on its own (one stump per lane, leaves added in stump
                // order via shuffles), so no block barrier is paid per stage.
                if (warp < n) {
                    const int idx = lists[(s & 1) * G::NW + warp];
                    const int wlx = idx % TX, wly = idx / TX;
                    const int b = wly * STEP * TW + wlx * STEP;
                    const float nfw = nfs[idx];
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
                            if (j < sd.n) leaf = eval_stage(T, b, nfw, grec, sd.first + j, 1, sd.mc);
                            const int m = min(32, sd.n - c0);
                            // ordered sum of the lanes' leaves: independent shuffles, serial adds
#pragma unroll
                            for (int t2 = 0; t2 < 32; ++t2) {
                                const float v = __shfl_sync(0xffffffffu, leaf, t2);
                                if (t2 < m) sum = __fadd_rn(sum, v);
                            }
                        }
                        if (!(sum >= sd.T)) break;
                    }
                    if (lane == 0) {
                        const long long o = (long long)frame * p.win_per_frame + L.win0 +
                                            (long long)(wy0 + wly) * L.nx + (wx0 + wlx);
                        if (s2 < N) {
                            if (DEPTH) {
                                p.depth[o] = (uint8_t)(s2 < 255 ? s2 : 255);
                                p.score[o] = sum;
                            }
                        } else {
                            if (p.stage_counts) atomicAdd(p.stage_counts + N, 1ull);
                            if (DEPTH) {
                                p.depth[o] = (uint8_t)(N < 255 ? N : 255);
                                p.score[o] = sum;
                            } else {
                                const unsigned long long at = atomicAdd(p.det_count, 1ull);
                                if ((long long)at < p.det_cap) {
                                    p.det_keys[at] = det_key(frame, k, (wy0 + wly) * STEP, (wx0 + wlx) * STEP);
                                    p.det_scores[at] = sum;
                                }
                            }
                        }
                    }
                }
                tail_done = true;
#ifdef FD_K2_TIMING
                if (lane == 0 && warp < n) {
                    atomicAdd(&g_k2_timing[80], (unsigned long long)(clock64() - ts0));
                    atomicAdd(&g_k2_timing[81], 1ull);
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
            __syncthreads();
#ifdef FD_K2_TIMING
            if (tid == 0) {
                const unsigned long long dt = (unsigned long long)(clock64() - ts0);
                const int si = s < 32 ? s : 31;
                atomicAdd(&g_k2_timing[16 + si], dt);
                atomicAdd(&g_k2_timing[48 + si], 1ull);
                atomicAdd(&g_k2_timing[n < p.lane_min ? 82 : 83], dt);
            }
#endif
        }
#ifdef FD_K2_TIMING
        if (tid == 0) {
            const long long tm3 = clock64();
            atomicAdd(&g_k2_timing[0], 1ull);
            atomicAdd(&g_k2_timing[1], (unsigned long long)(tm1 - tm0));
            atomicAdd(&g_k2_timing[2], (unsigned long long)(tm2 - tm1));
            atomicAdd(&g_k2_timing[3], (unsigned long long)(tm3 - tm2));
            atomicAdd(&g_k2_timing[4 + (s < 11 ? s : 11)], 1ull);
        }
#endif
        if (s == N && !tail_done) {                 // accepted windows: depth N
            const int nacc = s_cnt[N % 3];
            if (tid == 0 && p.stage_counts && nacc) atomicAdd(p.stage_counts + N, (unsigned long long)nacc);
            const uint16_t* lacc = lists + (N & 1) * G::NW;
            for (int e0 = warp * 32; e0 < nacc; e0 += G::THREADS) {
                const int e = e0 + lane;
                const bool act = e < nacc;
                int idx = act ? lacc[e] : 0;
                const int wlx = idx % TX, wly = idx / TX;
                if (DEPTH) {
                    if (act) {
                        const long long o = (long long)frame * p.win_per_frame + L.win0 +
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

#ifndef __CUDACC_RTC__
// TMA stages (FD_K2_STAGES=1|2, default 1: measured faster, 3 CTAs/SM hide more latency)
static int k2_stages() {
    static int v = [] {
        const char* e = getenv("FD_K2_STAGES");
        return (e && e[0] == '2') ? 2 : 1;
    }();
    return v;
}

template <int STEP, bool DEPTH, int NST>
static cudaError_t launch_one(const CascadeParams& p, int grid, cudaStream_t st) {
    const size_t smem = TileGeo<STEP>::smem(NST);
    cudaError_t e = cudaFuncSetAttribute(k_cascade<STEP, DEPTH, NST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_cascade<STEP, DEPTH, NST><<<grid, k2_threads(STEP), smem, st>>>(p);
    return cudaGetLastError();
}

template <int STEP, bool DEPTH, int NST>
static int grid_one() {
    const size_t smem = TileGeo<STEP>::smem(NST);
    cudaFuncSetAttribute(k_cascade<STEP, DEPTH, NST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_cascade<STEP, DEPTH, NST>, k2_threads(STEP), smem);
    return sms * (per > 0 ? per : 1);
}

template <int STEP, bool DEPTH>
static int grid_step() {
    return k2_stages() == 1 ? grid_one<STEP, DEPTH, 1>() : grid_one<STEP, DEPTH, 2>();
}

template <int STEP, bool DEPTH>
static cudaError_t launch_step(const CascadeParams& p, int grid, cudaStream_t st) {
    return k2_stages() == 1 ? launch_one<STEP, DEPTH, 1>(p, grid, st) : launch_one<STEP, DEPTH, 2>(p, grid, st);
}

size_t cascade_smem(int step) {
    const int n = k2_stages();
    switch (step) {
        case 1: return TileGeo<1>::smem(n);
        case 2: return TileGeo<2>::smem(n);
        case 3: return TileGeo<3>::smem(n);
        default: return TileGeo<4>::smem(n);
    }
}

int cascade_grid(bool depth, int step) {
    switch (step) {
        case 1: return depth ? grid_step<1, true>() : grid_step<1, false>();
        case 2: return depth ? grid_step<2, true>() : grid_step<2, false>();
        case 3: return depth ? grid_step<3, true>() : grid_step<3, false>();
        default: return depth ? grid_step<4, true>() : grid_step<4, false>();
    }
}

cudaError_t launch_cascade(const CascadeParams& p, bool depth, int step, int grid, cudaStream_t st) {
    switch (step) {
        case 1: return depth ? launch_step<1, true>(p, grid, st) : launch_step<1, false>(p, grid, st);
        case 2: return depth ? launch_step<2, true>(p, grid, st) : launch_step<2, false>(p, grid, st);
        case 3: return depth ? launch_step<3, true>(p, grid, st) : launch_step<3, false>(p, grid, st);
        case 4: return depth ? launch_step<4, true>(p, grid, st) : launch_step<4, false>(p, grid, st);
        default: return cudaErrorInvalidValue;
    }
}

#endif  // !__CUDACC_RTC__

}  // namespace fdk
