// k_cascade_ws.cu -- K2, warp-specialised pipeline (window step 1, the north_star workload).
//
// Same method and arithmetic as k_cascade.cu (stage 1 dense over every window, compacted deeper
// stages, oracle-exact fp32), scheduled as a Blackwell producer/consumer pipeline so that the
// latency-bound deep stages of one tile overlap the throughput-bound first stage of the next:
//
//   warp 16 (producer)  claims tiles from the global counter and issues two TMA loads per tile
//                       (ii plane into one of NSLOT slots, sqii plane into one of NSQ buffers);
//   warps 0-7 (dense)   stage 1 for all 2048 windows of tile i: nf from ii/sqii, survivors
//                       (window index + nf) appended to the slot's queue;
//   warps 8-11 / 12-15  two deep groups, alternating tiles: stages 2..N of tile i over the
//   (deep groups)       queue (lane-per-window, GL-lanes-per-window or warp-per-window modes),
//                       detections emitted, slot released.
//
// All hand-offs are mbarriers (full_ii, full_sq: TMA tx-count; dense_done; slot_free, sq_free),
// each guarded so no barrier runs more than one phase ahead of its consumer.  Named barriers
// (bar.sync 1..3) synchronise within the dense warps and within each deep group.
#include "k_common.cuh"

namespace fdk {
namespace wsk {

constexpr int TXW = 64, TYW = 32, WPT = 8;
constexpr int TW = tile_w(1), TH = tile_h(1);       // 88 x 56 ii values per tile
constexpr int PLANE = TW * TH;
constexpr int PLANE_BUF = (PLANE + 255) & ~255;     // 1 KB aligned stride
constexpr int NW = TXW * TYW;                       // 2048 windows per tile
constexpr int NSLOT = 4;                            // ii slots: dense i, deep i-1, deep i-2, TMA i+1
constexpr int NSQ = 2;                              // sqii buffers (first stage only)
constexpr int DENSE_WARPS = 8, DEEP_WARPS = 4, NGROUPS = 2;
constexpr int PRODUCER_WARP = DENSE_WARPS + NGROUPS * DEEP_WARPS;
constexpr int THREADS = 32 * (PRODUCER_WARP + 1);   // 544
constexpr int GL = 8, LEAF_CHUNK = 64;
constexpr int LEAVES_PER_GROUP = DEEP_WARPS * (32 / GL) * LEAF_CHUNK;
constexpr size_t OFF_II = 0;
constexpr size_t OFF_SQ = OFF_II + (size_t)NSLOT * PLANE_BUF * 4;
constexpr size_t OFF_LIDX = OFF_SQ + (size_t)NSQ * PLANE_BUF * 4;       // u16 [NSLOT][NW]
constexpr size_t OFF_LNF = OFF_LIDX + (size_t)NSLOT * NW * 2;           // f32 [NSLOT][NW]
constexpr size_t OFF_GIDX = OFF_LNF + (size_t)NSLOT * NW * 4;           // u16 [NGROUPS][NW]
constexpr size_t OFF_GNF = OFF_GIDX + (size_t)NGROUPS * NW * 2;         // f32 [NGROUPS][NW]
constexpr size_t OFF_LEAF = OFF_GNF + (size_t)NGROUPS * NW * 4;         // f32 [NGROUPS][LEAVES_PER_GROUP]
constexpr size_t SMEM = OFF_LEAF + (size_t)NGROUPS * LEAVES_PER_GROUP * 4;

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void named_bar(int id, int n) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}

template <bool DEPTH>
__global__ void __launch_bounds__(THREADS, 1) k_cascade_ws(const __grid_constant__ CascadeParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint32_t* ii_buf = reinterpret_cast<uint32_t*>(smem + OFF_II);
    uint32_t* sq_buf = reinterpret_cast<uint32_t*>(smem + OFF_SQ);
    uint16_t* lidx = reinterpret_cast<uint16_t*>(smem + OFF_LIDX);
    float* lnf = reinterpret_cast<float*>(smem + OFF_LNF);
    uint16_t* gidx = reinterpret_cast<uint16_t*>(smem + OFF_GIDX);
    float* gnf = reinterpret_cast<float*>(smem + OFF_GNF);
    float* leaves = reinterpret_cast<float*>(smem + OFF_LEAF);
    __shared__ __align__(8) uint64_t full_ii[NSLOT], full_sq[NSQ], dense_done[NSLOT], slot_free[NSLOT], sq_free[NSQ];
    __shared__ int slot_tile[NSLOT], slot_lvl[NSLOT], slot_tl[NSLOT], slot_n[NSLOT];
    __shared__ int grp_cnt[NGROUPS][3];

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int N = p.n_stages;
    if (tid == 0) {
        for (int i = 0; i < NSLOT; ++i) {
            mbar_init(&full_ii[i], 1);
            mbar_init(&dense_done[i], 1);
            mbar_init(&slot_free[i], 1);
            slot_n[i] = 0;
        }
        for (int i = 0; i < NSQ; ++i) {
            mbar_init(&full_sq[i], 1);
            mbar_init(&sq_free[i], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    // ================================================================ producer (one thread)
    if (warp == PRODUCER_WARP) {
        if (lane != 0) return;
        int sentinels = 0;
        for (int i = 0;; ++i) {
            const int slot = i % NSLOT, sqb = i % NSQ;
            if (i >= NSLOT) mbar_wait(&slot_free[slot], ((i / NSLOT) - 1) & 1);
            if (i >= NSQ) mbar_wait(&sq_free[sqb], ((i / NSQ) - 1) & 1);
            const int tn = sentinels ? p.total_tiles : (int)atomicAdd(p.tile_counter, 1u);
            if (tn >= p.total_tiles) {           // end of work: one sentinel per deep group
                slot_tile[slot] = -1;
                mbar_arrive(&full_ii[slot]);
                mbar_arrive(&full_sq[sqb]);
                if (++sentinels == NGROUPS) break;
                continue;
            }
            const int g = tn / p.tiles_per_frame, r = tn % p.tiles_per_frame;
            int k = 0;
            while (k + 1 < p.n_levels && __ldg(&p.lv[k + 1].tile0) <= r) ++k;
            const int tl = r - __ldg(&p.lv[k].tile0);
            const int tx = __ldg(&p.lv[k].tiles_x);
            slot_tile[slot] = tn;
            slot_lvl[slot] = k;
            slot_tl[slot] = tl;
            const int x = (tl % tx) * TXW, y = (tl / tx) * TYW;
            mbar_expect_tx(&full_ii[slot], PLANE * 4);
            tma_load_4d(ii_buf + slot * PLANE_BUF, p.tmaps + k, x, y, 0, g, &full_ii[slot]);
            mbar_expect_tx(&full_sq[sqb], PLANE * 4);
            tma_load_4d(sq_buf + sqb * PLANE_BUF, p.tmaps + k, x, y, 1, g, &full_sq[sqb]);
        }
        return;
    }

    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};

    // result of one window: depth d (stages passed) and the last evaluated stage sum
    auto finish = [&](int frame, int k, const LevelDev& L, int wx0, int wy0, int idx, int d, float score) {
        const int wlx = idx % TXW, wly = idx / TXW;
        if (d == N && p.stage_counts) atomicAdd(p.stage_counts + N, 1ull);
        if (DEPTH) {
            const long long o = (long long)frame * p.win_per_frame + L.win0 + (long long)(wy0 + wly) * L.nx + (wx0 + wlx);
            p.depth[o] = (uint8_t)(d < 255 ? d : 255);
            p.score[o] = score;
        } else if (d == N) {
            const unsigned long long at = atomicAdd(p.det_count, 1ull);
            if ((long long)at < p.det_cap) {
                p.det_keys[at] = det_key(frame, k, wy0 + wly, wx0 + wlx);
                p.det_scores[at] = score;
            }
        }
    };

    // ================================================================ dense warps: stage 1
    if (warp < DENSE_WARPS) {
        const StageDev& st0 = p.pstages[0];
        int sentinels = 0;
        for (int i = 0;; ++i) {
            const int slot = i % NSLOT, sqb = i % NSQ;
            mbar_wait(&full_ii[slot], (i / NSLOT) & 1);
            mbar_wait(&full_sq[sqb], (i / NSQ) & 1);
            const int t = slot_tile[slot];
            if (t < 0) {
                named_bar(1, DENSE_WARPS * 32);
                if (tid == 0) {
                    mbar_arrive(&dense_done[slot]);
                    mbar_arrive(&sq_free[sqb]);
                }
                if (++sentinels == NGROUPS) break;
                continue;
            }
            const int g = t / p.tiles_per_frame;
            const int k = slot_lvl[slot];
            const LevelDev L = p.lv[k];
            const int tl = slot_tl[slot];
            const int wx0 = (tl % L.tiles_x) * TXW, wy0 = (tl / L.tiles_x) * TYW;
            const int frame = p.frame_base + g;
            const uint32_t* T = ii_buf + slot * PLANE_BUF;
            const uint32_t* Q = sq_buf + sqb * PLANE_BUF;
            uint16_t* qidx = lidx + slot * NW;
            float* qnf = lnf + slot * NW;

            const int lx = lane + 32 * (warp & 1);
            const int ly0 = (warp >> 1) * WPT;
            const int base = ly0 * TW + lx;
            const bool colok = wx0 + lx < L.nx;
            float nf[WPT], sm[WPT];
#pragma unroll
            for (int w = 0; w < WPT; ++w) {
                const int b = base + w * TW;
                const uint32_t S = T[b + WIN * TW + WIN] - T[b + WIN] - T[b + WIN * TW] + T[b];
                const uint32_t q = Q[b + WIN * TW + WIN] - Q[b + WIN] - Q[b + WIN * TW] + Q[b];
                const long long v = 576LL * (long long)q - (long long)S * (long long)S;
                nf[w] = v > 0 ? __fsqrt_rn(__ll2float_rn(v)) : 1.0f;
                sm[w] = 0.0f;
            }
            if (st0.first + st0.n <= p.n_pstumps)
                dense_stage<WPT, TW>(T, base, nf, sm, prec, st0.first, st0.n);
            else
                dense_stage<WPT, TW>(T, base, nf, sm, grec, st0.first, st0.n);
#pragma unroll
            for (int w = 0; w < WPT; ++w) {
                const int wy = wy0 + ly0 + w;
                const bool valid = colok && wy < L.ny;
                const bool pass = valid && (sm[w] >= st0.T);
                const int idx = (ly0 + w) * TXW + lx;
                if (valid && (!pass || N == 1) && (DEPTH || pass)) finish(frame, k, L, wx0, wy0, idx, pass ? 1 : 0, sm[w]);
                const unsigned m = __ballot_sync(0xffffffffu, pass && N > 1);
                if (m) {
                    int pos = 0;
                    if (lane == 0) pos = atomicAdd(&slot_n[slot], __popc(m));
                    pos = __shfl_sync(0xffffffffu, pos, 0);
                    if (pass) {
                        const int at = pos + __popc(m & ((1u << lane) - 1u));
                        qidx[at] = (uint16_t)idx;
                        qnf[at] = nf[w];
                    }
                }
            }
            if (tid == 0 && p.stage_counts)
                atomicAdd(p.stage_counts,
                          (unsigned long long)min(TXW, L.nx - wx0) * (unsigned long long)min(TYW, L.ny - wy0));
            named_bar(1, DENSE_WARPS * 32);          // queue complete, sqii buffer consumed
            if (tid == 0) {
                mbar_arrive(&dense_done[slot]);
                mbar_arrive(&sq_free[sqb]);
            }
        }
        return;
    }

    // ================================================================ deep groups: stages 2..N
    const int grp = (warp - DENSE_WARPS) / DEEP_WARPS;          // 0 or 1
    const int gw = (warp - DENSE_WARPS) % DEEP_WARPS;           // warp within the group
    const int gtid = gw * 32 + lane;
    const int barid = 2 + grp;
    float* gleaves = leaves + grp * LEAVES_PER_GROUP;
    for (int i = grp;; i += NGROUPS) {
        const int slot = i % NSLOT;
        mbar_wait(&dense_done[slot], (i / NSLOT) & 1);
        const int t = slot_tile[slot];
        if (t < 0) break;
        const int g = t / p.tiles_per_frame;
        const int k = slot_lvl[slot];
        const LevelDev L = p.lv[k];
        const int tl = slot_tl[slot];
        const int wx0 = (tl % L.tiles_x) * TXW, wy0 = (tl / L.tiles_x) * TYW;
        const int frame = p.frame_base + g;
        const uint32_t* T = ii_buf + slot * PLANE_BUF;
        // ping-pong queues: odd stages read the slot queue, even stages the group queue
        uint16_t* const qg = gidx + grp * NW;
        uint16_t* const qs = lidx + slot * NW;
        float* const fg = gnf + grp * NW;
        float* const fs = lnf + slot * NW;
        if (gtid == 0) {
            grp_cnt[grp][1] = slot_n[slot];
            grp_cnt[grp][2] = 0;
            grp_cnt[grp][0] = 0;
        }
        named_bar(barid, DEEP_WARPS * 32);
        for (int s = 1; s < N; ++s) {
            const int n = grp_cnt[grp][s % 3];
            if (gtid == 0 && p.stage_counts && n) atomicAdd(p.stage_counts + s, (unsigned long long)n);
            if (n == 0) break;
            const bool odd = s & 1;
            const uint16_t* lin = odd ? qs : qg;
            const float* lnfi = odd ? fs : fg;
            uint16_t* lout = odd ? qg : qs;
            float* lnfo = odd ? fg : fs;
            if (n <= DEEP_WARPS) {
                // tail: one window per warp walks all remaining stages (no group barriers)
                if (gw < n) {
                    const int idx = lin[gw];
                    const float nfw = lnfi[gw];
                    const int b = (idx / TXW) * TW + (idx % TXW);
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
#pragma unroll
                            for (int t2 = 0; t2 < 32; ++t2) {
                                const float v = __shfl_sync(0xffffffffu, leaf, t2);
                                if (t2 < m) sum = __fadd_rn(sum, v);
                            }
                        }
                        if (!(sum >= sd.T)) break;
                    }
                    if (lane == 0 && (DEPTH || s2 == N)) finish(frame, k, L, wx0, wy0, idx, s2, sum);
                }
                break;
            }
            if (gtid == 0) grp_cnt[grp][(s + 2) % 3] = 0;
            StageDev sd;
            if (s < p.n_pstages) {
                sd.first = p.pstages[s].first;
                sd.n = p.pstages[s].n;
                sd.T = p.pstages[s].T;
                sd.mc = p.pstages[s].mc;
            } else {
                sd = p.stages[s];
            }
            const bool last = s == N - 1;
            if (n < p.lane_min) {
                // GL lanes per window (one stump per lane), leaves added in stump order
                const int sub = lane / GL, q = lane % GL;
                float* lv = gleaves + (gw * (32 / GL) + sub) * LEAF_CHUNK;
                for (int e0 = gw * (32 / GL); e0 < n; e0 += DEEP_WARPS * (32 / GL)) {
                    const int e = e0 + sub;
                    const bool act = e < n;
                    const int idx = act ? lin[e] : 0;
                    const float nfw = act ? lnfi[e] : 1.0f;
                    const int b = (idx / TXW) * TW + (idx % TXW);
                    float sum = 0.0f;
                    for (int c0 = 0; c0 < sd.n; c0 += LEAF_CHUNK) {
                        const int cn = min(LEAF_CHUNK, sd.n - c0);
                        if (act)
                            for (int j = q; j < cn; j += GL) lv[j] = eval_stage(T, b, nfw, grec, sd.first + c0 + j, 1, sd.mc);
                        __syncwarp();
                        if (act && q == 0) {
                            int t2 = 0;
                            for (; t2 + 8 <= cn; t2 += 8) {
                                const float4 a = *reinterpret_cast<const float4*>(lv + t2);
                                const float4 c = *reinterpret_cast<const float4*>(lv + t2 + 4);
                                sum = __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(sum, a.x), a.y), a.z), a.w);
                                sum = __fadd_rn(__fadd_rn(__fadd_rn(__fadd_rn(sum, c.x), c.y), c.z), c.w);
                            }
                            for (; t2 < cn; ++t2) sum = __fadd_rn(sum, lv[t2]);
                        }
                        __syncwarp();
                    }
                    if (act && q == 0) {
                        const bool pass = sum >= sd.T;
                        if (pass && !last) {
                            const int at = atomicAdd(&grp_cnt[grp][(s + 1) % 3], 1);
                            lout[at] = (uint16_t)idx;
                            lnfo[at] = nfw;
                        } else if (DEPTH || pass) {
                            finish(frame, k, L, wx0, wy0, idx, pass ? N : s, sum);
                        }
                    }
                }
            } else {
                const bool in_param = sd.first + sd.n <= p.n_pstumps;
                for (int e0 = gw * 32; e0 < n; e0 += DEEP_WARPS * 32) {
                    const int e = e0 + lane;
                    const bool act = e < n;
                    int idx = 0;
                    float nfw = 1.0f, sum = 0.0f;
                    if (act) {
                        idx = lin[e];
                        nfw = lnfi[e];
                        const int b = (idx / TXW) * TW + (idx % TXW);
                        sum = in_param ? eval_stage(T, b, nfw, prec, sd.first, sd.n, sd.mc)
                                       : eval_stage(T, b, nfw, grec, sd.first, sd.n, sd.mc);
                    }
                    const bool pass = act && (sum >= sd.T);
                    if (act && (!pass || last) && (DEPTH || pass)) finish(frame, k, L, wx0, wy0, idx, pass ? N : s, sum);
                    const unsigned m = __ballot_sync(0xffffffffu, pass && !last);
                    if (m) {
                        int pos = 0;
                        if (lane == 0) pos = atomicAdd(&grp_cnt[grp][(s + 1) % 3], __popc(m));
                        pos = __shfl_sync(0xffffffffu, pos, 0);
                        if (pass) {
                            const int at = pos + __popc(m & ((1u << lane) - 1u));
                            lout[at] = (uint16_t)idx;
                            lnfo[at] = nfw;
                        }
                    }
                }
            }
            named_bar(barid, DEEP_WARPS * 32);
        }
        named_bar(barid, DEEP_WARPS * 32);           // all deep work of the tile done
        if (gtid == 0) {
            slot_n[slot] = 0;
            mbar_arrive(&slot_free[slot]);
        }
    }
}

}  // namespace wsk

size_t cascade_ws_smem() { return wsk::SMEM; }

cudaError_t launch_cascade_ws(const CascadeParams& p, bool depth, cudaStream_t st) {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = sms < p.total_tiles ? sms : p.total_tiles;
    cudaError_t e;
    if (depth) {
        e = cudaFuncSetAttribute(wsk::k_cascade_ws<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)wsk::SMEM);
        if (e != cudaSuccess) return e;
        wsk::k_cascade_ws<true><<<grid, wsk::THREADS, wsk::SMEM, st>>>(p);
    } else {
        e = cudaFuncSetAttribute(wsk::k_cascade_ws<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)wsk::SMEM);
        if (e != cudaSuccess) return e;
        wsk::k_cascade_ws<false><<<grid, wsk::THREADS, wsk::SMEM, st>>>(p);
    }
    return cudaGetLastError();
}

}  // namespace fdk
