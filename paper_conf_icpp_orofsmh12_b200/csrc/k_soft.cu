// k_soft.cu -- K2 for a soft cascade (the paper's future work, P:L1685-1687,
// ref [32]; reading R8b): the stage sum is not restarted at a stage boundary, it runs
// over every stump evaluated so far (fp32, stump order) and T_s is the rejection threshold of
// that running sum after stage s.  One-stump stages give the per-stump rejection trace of [32].
//
// The hard-cascade schedules (k_stage1 / k_deep1 / k_tail) compact survivors between stages and
// restart every sum at 0; a soft cascade would have to carry a running sum per survivor through
// all of them.  This kernel is a separate, self-contained schedule instead:
//   * persistent over every (frame, level, tile) of a frame group (atomic tile counter), the
//     same 64 x 32-window tiles and the same TMA of the tile's ii and sqii planes as k_cascade;
//   * stage 0 is dense, as in k_cascade: each thread owns WPT windows down one column, stump
//     records from the kernel-parameter bank (warp-uniform); its survivors (c3: ~6%) are
//     ballot-compacted into a shared list with their nf and running sum;
//   * stages 1..N-1 run over that list one lane per window; a lane takes the next window from the
//     list (shared atomic) as soon as its current one is rejected or accepted, so lanes idle only
//     once the list is drained, and no block barrier separates the stages;
//   * leaves are added with __fadd_rn in stump order -- the definition's fp32 sequence -- so
//     scores and depths are bit-identical to the oracle.  Stage counters are kept per CTA in
//     shared memory and flushed once at exit.
#include "k_common.cuh"

namespace fdk {

constexpr int SOFT_MAX_STAGES = 256;      // the .fdc parser allows at most 250 stages

template <int STEP, bool DEPTH, bool SOFT>
__global__ void __launch_bounds__(k2_threads(STEP), 2) k_soft(const __grid_constant__ CascadeParams p) {
    using G = TileGeo<STEP>;
    constexpr int TW = tile_w(STEP), TX = k2_tx(STEP), TY = k2_ty(STEP), WPT = k2_wpt(STEP), NW = G::NW;
    constexpr int WARPS_X = TX / 32, PLANE = tile_w(STEP) * tile_h(STEP);
    static_assert(G::SMEM >= G::OFF_Q + (size_t)NW * 10, "survivor list must fit in the sqii buffer");
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint32_t* T = reinterpret_cast<uint32_t*>(smem_raw);                      // ii plane
    uint32_t* Q = reinterpret_cast<uint32_t*>(smem_raw + G::OFF_Q);           // sqii plane (mod 2^32)
    // stage-0 survivors, over the sqii buffer once every nf is taken: nf, running sum, window
    float* l_nf = reinterpret_cast<float*>(smem_raw + G::OFF_Q);
    float* l_sum = reinterpret_cast<float*>(smem_raw + G::OFF_Q + (size_t)NW * 4);
    uint16_t* l_idx = reinterpret_cast<uint16_t*>(smem_raw + G::OFF_Q + (size_t)NW * 8);
    __shared__ __align__(8) uint64_t mbar;
    __shared__ int s_tile, s_frame, s_lvl, s_wx0, s_wy0, s_cnt, s_next;
    __shared__ unsigned s_sc[SOFT_MAX_STAGES + 1];                            // stage entry counts of a tile
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};
    const StageDev& st0 = p.pstages[0];
    const int N = p.n_stages;
    const bool counting = p.stage_counts != nullptr;
    if (tid == 0) {
        mbar_init(&mbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (counting)
        for (int i = tid; i <= N; i += blockDim.x) s_sc[i] = 0;
    uint32_t phase = 0;
    for (;;) {
        __syncthreads();                          // buffers and s_* free
        if (tid == 0) {
            const int tn = (int)atomicAdd(p.tile_counter, 1u);
            s_tile = tn;
            s_cnt = 0;
            s_next = 0;
            if (tn < p.total_tiles) {
                const int g = tn / p.tiles_per_frame, r = tn % p.tiles_per_frame;
                int k = 0;
                while (k + 1 < p.n_levels && __ldg(&p.lv[k + 1].tile0) <= r) ++k;
                const int tl = r - __ldg(&p.lv[k].tile0), tx = __ldg(&p.lv[k].tiles_x);
                s_frame = p.frame_base + g;
                s_lvl = k;
                s_wx0 = (tl % tx) * TX;
                s_wy0 = (tl / tx) * TY;
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_expect_tx(&mbar, 2 * PLANE * 4);
                tma_load_4d(T, p.tmaps + k, s_wx0 * STEP, s_wy0 * STEP, 0, g, &mbar);
                tma_load_4d(Q, p.tmaps + k, s_wx0 * STEP, s_wy0 * STEP, 1, g, &mbar);
            }
        }
        __syncthreads();
        if (s_tile >= p.total_tiles) break;
        mbar_wait(&mbar, phase);
        phase ^= 1;
        const int k = s_lvl, frame = s_frame, wx0 = s_wx0, wy0 = s_wy0;
        const int nx = __ldg(&p.lv[k].nx), ny = __ldg(&p.lv[k].ny);
        const long long lvl_win0 = (long long)frame * p.win_per_frame + __ldg(&p.lv[k].win0);
        const int lx = lane + 32 * (warp % WARPS_X);
        const int ly0 = (warp / WARPS_X) * WPT;
        const int base = ly0 * STEP * TW + lx * STEP;
        const bool colok = wx0 + lx < nx;
        // a window leaves the cascade: depth map entry or detection (running sum = score)
        auto finish = [&](int idx, int depth, float sum) {
            const int wy = wy0 + idx / TX, wx = wx0 + idx % TX;
            if (DEPTH) {
                const long long o = lvl_win0 + (long long)wy * nx + wx;
                p.depth[o] = (uint8_t)(depth < 255 ? depth : 255);
                p.score[o] = sum;
            } else if (depth == N) {
                const unsigned long long at = atomicAdd(p.det_count, 1ull);
                if ((long long)at < p.det_cap) {
                    p.det_keys[at] = det_key(frame, k, wy * STEP, wx * STEP);
                    p.det_scores[at] = sum;
                }
            }
        };
        // stage 0, dense: every window of the tile, WPT per thread down a column (as k_cascade)
        float nf[WPT], sm[WPT];
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const int b = base + i * STEP * TW;
            const uint32_t S = T[b + WIN * TW + WIN] - T[b + WIN] - T[b + WIN * TW] + T[b];
            const uint32_t q = Q[b + WIN * TW + WIN] - Q[b + WIN] - Q[b + WIN * TW] + Q[b];
            const long long v = 576LL * (long long)q - (long long)S * (long long)S;
            nf[i] = v > 0 ? __fsqrt_rn(__ll2float_rn(v)) : 1.0f;
            sm[i] = 0.0f;
        }
        if (st0.first + st0.n <= p.n_pstumps)
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, prec, st0.first, st0.n);
        else
            dense_stage<WPT, STEP * TW>(T, base, nf, sm, grec, st0.first, st0.n);
        __syncthreads();                          // every sqii read done: the buffer becomes the list
#pragma unroll
        for (int i = 0; i < WPT; ++i) {
            const bool valid = colok && wy0 + ly0 + i < ny;
            const bool pass = valid && sm[i] >= st0.T;
            const int idx = (ly0 + i) * TX + lx;
            if (valid && (!pass || N == 1)) finish(idx, pass ? 1 : 0, sm[i]);
            if (N == 1) {
                const unsigned m = __ballot_sync(0xffffffffu, pass);
                if (counting && lane == 0 && m) atomicAdd(&s_sc[1], (unsigned)__popc(m));
                continue;
            }
            const unsigned m = __ballot_sync(0xffffffffu, pass);
            if (m) {
                int pos = 0;
                if (lane == 0) pos = atomicAdd(&s_cnt, __popc(m));
                pos = __shfl_sync(0xffffffffu, pos, 0);
                if (pass) {
                    const int at = pos + __popc(m & ((1u << lane) - 1u));
                    l_idx[at] = (uint16_t)idx;
                    l_nf[at] = nf[i];
                    l_sum[at] = sm[i];
                }
            }
        }
        if (tid == 0 && counting)
            atomicAdd(p.stage_counts, (unsigned long long)min(TX, nx - wx0) * (unsigned long long)min(TY, ny - wy0));
        __syncthreads();                          // list complete
        // stages 1 .. N-1 over the list: each lane takes the next window whenever it is free and
        // carries that window's running sum across the stage boundaries (R8b)
        const int cnt = s_cnt;
        int e = -1, s = 0, b = 0, idx = 0;
        float sum = 0.0f, nfw = 1.0f;
        bool alive = false;
        for (;;) {
            if (!alive) {
                e = atomicAdd(&s_next, 1);
                if (e < cnt) {
                    idx = l_idx[e];
                    nfw = l_nf[e];
                    sum = l_sum[e];
                    b = (idx / TX) * STEP * TW + (idx % TX) * STEP;
                    s = 1;
                    alive = true;
                }
            }
            if (!__any_sync(0xffffffffu, alive)) break;
            if (!alive) continue;
            const StageDev sd = s < p.n_pstages ? p.pstages[s] : p.stages[s];
            if (counting) atomicAdd(&s_sc[s], 1u);
            if (!SOFT) sum = 0.0f;                // hard cascade (R8): every stage sum starts at 0
            for (int j = sd.first; j < sd.first + sd.n; ++j)
                sum = __fadd_rn(sum, eval_stump_mc<MAX_CORNERS>(T, b, nfw, grec, j));
            const bool pass = sum >= sd.T;
            if (pass && s + 1 < N) {
                ++s;
                continue;
            }
            alive = false;
            if (pass && counting) atomicAdd(&s_sc[N], 1u);
            finish(idx, pass ? N : s, sum);
        }
    }
    if (counting) {
        __syncthreads();
        for (int i = tid; i <= N; i += blockDim.x)
            if (i > 0 && s_sc[i]) atomicAdd(p.stage_counts + i, (unsigned long long)s_sc[i]);
    }
}

template <int STEP, bool DEPTH, bool SOFT>
static cudaError_t launch_soft_t(const CascadeParams& p, cudaStream_t st) {
    const size_t smem = TileGeo<STEP>::SMEM;
    cudaError_t e = cudaFuncSetAttribute(k_soft<STEP, DEPTH, SOFT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_soft<STEP, DEPTH, SOFT>, k2_threads(STEP), smem);
    int grid = sms * (per > 0 ? per : 1);
    if (grid > p.total_tiles) grid = p.total_tiles;
    k_soft<STEP, DEPTH, SOFT><<<grid, k2_threads(STEP), smem, st>>>(p);
    return cudaGetLastError();
}

template <bool SOFT>
static cudaError_t launch_q(const CascadeParams& p, bool depth, int step, cudaStream_t st) {
    switch (step) {
        case 1: return depth ? launch_soft_t<1, true, SOFT>(p, st) : launch_soft_t<1, false, SOFT>(p, st);
        case 2: return depth ? launch_soft_t<2, true, SOFT>(p, st) : launch_soft_t<2, false, SOFT>(p, st);
        case 3: return depth ? launch_soft_t<3, true, SOFT>(p, st) : launch_soft_t<3, false, SOFT>(p, st);
        case 4: return depth ? launch_soft_t<4, true, SOFT>(p, st) : launch_soft_t<4, false, SOFT>(p, st);
        default: return cudaErrorInvalidValue;
    }
}

// soft = true: a soft cascade (R8b); false: a hard cascade on the same queue schedule
// (FD_K2_QUEUE=1, an alternative K2 schedule measured against the default)
cudaError_t launch_soft(const CascadeParams& p, bool depth, int step, bool soft, cudaStream_t st) {
    return soft ? launch_q<true>(p, depth, step, st) : launch_q<false>(p, depth, step, st);
}

}  // namespace fdk
