// k_deepq.cuh -- K2b, the deep stages (s0 .. N-1) as warp-autonomous batches over a per-SM pool of
// tiles (included by k_cascade.cu; also compiled by NVRTC with the cascade's specialised stages).
//
// The paper evaluates the deeper stages in the thread that owns the window, so warps empty out as
// windows are rejected (the divergence problem; Fig. 7's rejection profile,
// P:L1311-1325).  k_stage1 leaves ~1.7% of the windows alive after stage 2, ~70 per tile that has
// any.  Here one persistent CTA per SM keeps NS tiles' ii planes in shared memory (TMA, one
// mbarrier per slot, with the tile's survivor list copied next to it) and every warp works on
// its own batch of up to 32 windows -- fresh stage-s0 windows of any loaded tiles, one lane per
// window, so the stump records stay warp-uniform (parameter bank / generated code):
//   * after each stage the warp compacts its survivors (ballot + rank) and goes on with them; a
//     batch of at most FD_DQ_GROUP windows runs GL = 2^lg lanes per window (the largest with
//     cnt * GL <= 32) that share the stage's stumps, so a thinning batch keeps its lanes busy and
//     its latency short;
//   * windows entering stage s_tail leave for k_tail's queue (one warp per window there): the
//     long chains of the last stages would otherwise hold their tile's slot;
//   * when its batch is empty the warp takes fresh windows (a CAS on the slot's taken | n word)
//     or claims a prefetched tile into a free slot; there is no CTA barrier after the start and
//     no lock, so a tile's slowest window never holds up the others;
//   * a slot is reloaded once every window of its tile has finished (per-slot alive count).
// Windows of different tiles share a batch (each lane addresses its own slot's plane).  Decisions,
// scores and outputs are the definition's: sequential fp32 stage sums in stump order, or tree
// sums whose decision is certified against their rounding bound (oracle c7/c8).
#pragma once

namespace fdk {

#ifndef FD_JIT_DEEPQ
#define FD_JIT_DEEPQ 0       // run-time specialised kernel: stages [1, FD_JIT_DEEPQ) are generated code
#endif
#ifndef FD_DQ_NPF
#define FD_DQ_NPF 4             // tile-list entries prefetched per CTA
#endif
#ifndef FD_DQ_GROUP
#define FD_DQ_GROUP 16          // batches of at most this many windows run GL > 1 lanes per window
#endif

// Compact evaluators (one stump per loop iteration, the corner count padded to 9 or 12 with zero
// corners): every warp of the SM runs its own stage, so the code they execute together must stay
// inside the instruction caches (L0 ~6 KB, L1.5 32 KB per SM) -- unrolled variants per corner count
// made k_deepq's warps wait on instruction fetch more than on anything else.
template <int MC, class R>
__device__ __forceinline__ float dq_stage_mc(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int first,
                                         int n) {
    float sum = 0.0f;
#pragma unroll 1
    for (int j = first; j < first + n; ++j) sum = __fadd_rn(sum, eval_stump_mc<MC>(T, b, nf, rec, j));
    return sum;
}
template <class R>
__device__ __forceinline__ float dq_stage(const uint32_t* __restrict__ T, int b, float nf, const R& rec, int first, int n,
                                          int mc) {
    return mc <= 9 ? dq_stage_mc<9>(T, b, nf, rec, first, n) : dq_stage_mc<MAX_CORNERS>(T, b, nf, rec, first, n);
}
// GL = 2^lg lanes per window: lane q takes stumps q, q + GL, ...; sum and sum of magnitudes of its
// leaves, then the group's butterfly (k_common.cuh group_stage_tree, without its unrolling)
template <int MC>
__device__ __forceinline__ float2 dq_group_mc(const uint32_t* __restrict__ T, int b, float nf, const uint4* __restrict__ st,
                                          int first, int n, int lg, bool act, int lane) {
    const int gl = 1 << lg, q = lane & (gl - 1);
    const GlobalRec rec{st};
    float acc = 0.0f, aacc = 0.0f;
    if (act) {
#pragma unroll 1
        for (int j = q; j < n; j += gl) {
            const float l = eval_stump_mc<MC>(T, b, nf, rec, first + j);
            acc = __fadd_rn(acc, l);
            aacc = __fadd_rn(aacc, fabsf(l));
        }
    }
    for (int o = gl >> 1; o > 0; o >>= 1) {
        acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, o));
        aacc = __fadd_rn(aacc, __shfl_xor_sync(0xffffffffu, aacc, o));
    }
    return make_float2(acc, aacc);
}

template <int STEP, bool DEPTH>
__global__ void __launch_bounds__(DQ_THREADS, 1) k_deepq(const __grid_constant__ CascadeParams p) {
    using G = TileGeoQ<STEP>;
    constexpr int TX = k2_tx(STEP), TW = tile_w(STEP), PBUF = G::PBUF, PLANE = tile_w(STEP) * tile_h(STEP);
    constexpr int NS = G::NS, NPF = FD_DQ_NPF, CAPF = DQ_CAPF;
    constexpr unsigned ALL = (NS == 32) ? 0xffffffffu : ((1u << NS) - 1u);
    constexpr unsigned FULL = 0xffffffffu;
    static_assert(NPF <= 32, "one lane per prefetch entry");
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    const uint32_t* planes = reinterpret_cast<const uint32_t*>(smem_raw);
    uint2* flist = reinterpret_cast<uint2*>(smem_raw + G::OFF_F);                  // [NS][CAPF] {window, nf bits}
    uint2* stg = reinterpret_cast<uint2*>(smem_raw + G::OFF_STG) + (threadIdx.x >> 5) * 32;   // this warp's
    __shared__ __align__(8) uint64_t mbar[NS];
    __shared__ int s_frame[NS], s_lvl[NS], s_wx0[NS], s_wy0[NS];
    __shared__ int s_alive[NS];             // windows of the slot's tile not finished yet
    __shared__ unsigned s_fw[NS];           // fresh windows: taken << 16 | n (taken == n: none left)
    __shared__ int s_foff[NS];              // the tile's survivors: p.surv[foff, foff + n), first CAPF in flist
    __shared__ int s_wpar[NS];              // mbarrier parity of the slot's current load
    __shared__ unsigned s_free;
    __shared__ int s_pfst[NPF];             // prefetched tile-list entries: 0 filling, 1 owned, 2 ready, 3 none left
    __shared__ int4 s_pf0[NPF], s_pf1[NPF]; // {tile, off, n, -}, {g, k, wx0, wy0}
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int N = p.n_stages, s0 = p.s0;
    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};
    const WinOut<STEP, DEPTH> out{p, s_frame, s_lvl, s_wx0, s_wy0};
    volatile int* vpfst = s_pfst;
    volatile unsigned* vfw = s_fw;
    volatile unsigned* vfree = &s_free;
    // prefetch entry i: the next tile with stage-s0 survivors (one lane, no lock; the entry is
    // owned by the caller until its state becomes 2 or 3)
    auto refill = [&](int i) {
        const unsigned li = atomicAdd(p.deep_counter, 1u);
        const unsigned nl = *reinterpret_cast<volatile const unsigned*>(p.tile_list_count);
        if (li < nl) {
            const uint4 e = p.tile_list[li];
            const TileAt t = tile_at<STEP>(p, (int)e.x);
            s_pf0[i] = make_int4((int)e.x, (int)e.y, (int)e.z, 0);
            s_pf1[i] = make_int4(t.g, t.k, t.wx0, t.wy0);
            __threadfence_block();
            vpfst[i] = 2;
        } else {
            vpfst[i] = 3;
        }
    };
    if (tid == 0) {
        for (int i = 0; i < NS; ++i) mbar_init(&mbar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        s_free = ALL;
    }
    if (tid < NS) {
        s_alive[tid] = 0;
        s_fw[tid] = 0u;
        s_wpar[tid] = 0;
    }
    if (tid < NPF) s_pfst[tid] = 0;
    __syncthreads();
    if (lane == 0 && warp < NPF) refill(warp);

    // fresh windows of slot sl into lanes [dst, dst + got), at most k; warp-uniform result
    auto take_fresh = [&](int sl, int k, int dst, uint32_t& loc, float& nf) -> int {
        int t0 = 0, got = 0;
        if (lane == 0) {
            for (;;) {
                const unsigned w = vfw[sl];
                const int taken = (int)(w >> 16), n = (int)(w & 0xffffu);
                const int t = min(k, n - taken);
                if (t <= 0) break;
                if (atomicCAS(&s_fw[sl], w, ((unsigned)(taken + t) << 16) | (unsigned)n) == w) {
                    t0 = taken;
                    got = t;
                    break;
                }
            }
        }
        got = __shfl_sync(FULL, got, 0);
        t0 = __shfl_sync(FULL, t0, 0);
        if (lane >= dst && lane < dst + got) {
            __threadfence_block();
            const int j = t0 + lane - dst;
            const uint2 v = j < CAPF ? flist[sl * CAPF + j] : p.surv[*reinterpret_cast<volatile int*>(&s_foff[sl]) + j];
            loc = ((uint32_t)sl << 16) | v.x;
            nf = __uint_as_float(v.y);
        }
        return got;
    };
    // claim a prefetched tile into a free slot (TMA of its ii plane, its survivor list copied by
    // the warp); the slot index or -1.  Warp-collective.
    auto claim = [&]() -> int {
        int sl = -1, pf = -1;
        if (lane == 0) {
            for (int i = 0; i < NPF && pf < 0; ++i)
                if (vpfst[i] == 2 && atomicCAS(&s_pfst[i], 2, 1) == 2) pf = i;
            if (pf >= 0) {
                for (;;) {
                    const unsigned m = *vfree;
                    if (!m) break;
                    const unsigned bit = m & (0u - m);
                    if (atomicAnd(&s_free, ~bit) & bit) {
                        sl = __ffs(bit) - 1;
                        break;
                    }
                }
                if (sl < 0) {
                    vpfst[pf] = 2;                           // no slot after all: give the entry back
                } else {
                    __threadfence_block();
                    const int4 a = s_pf0[pf], b = s_pf1[pf];
                    s_frame[sl] = p.frame_base + b.x;
                    s_lvl[sl] = b.y;
                    s_wx0[sl] = b.z;
                    s_wy0[sl] = b.w;
                    s_alive[sl] = a.z;
                    s_foff[sl] = a.y;
                    const int par = s_wpar[sl] ^ 1;          // the slot's loads alternate parities
                    s_wpar[sl] = par;
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    mbar_expect_tx(&mbar[sl], PLANE * 4);
                    tma_load_4d(const_cast<uint32_t*>(planes) + sl * PBUF, p.tmaps + b.y, b.z * STEP, b.w * STEP, 0,
                                b.x, &mbar[sl]);
                }
            }
        }
        sl = __shfl_sync(FULL, sl, 0);
        pf = __shfl_sync(FULL, pf, 0);
        if (sl >= 0) {
            __syncwarp();
            const int off = s_foff[sl], n = s_alive[sl];     // written by lane 0 above
            for (int j = lane; j < min(n, CAPF); j += 32) flist[sl * CAPF + j] = p.surv[off + j];
            __syncwarp();
            if (lane == 0) {
                __threadfence_block();
                vfw[sl] = (unsigned)n;                       // publish: 0 taken of n
                refill(pf);
            }
        }
        return sl;
    };

    int cnt = 0, s = s0;          // this warp's batch: lanes [0, cnt) hold windows entering stage s
    uint32_t loc = 0;             // slot << 16 | window index within the slot's tile
    float nf = 1.0f;
    int backoff = 64;
    for (;;) {
        if (cnt == 0) {
            // ---------------- new batch: fresh windows of loaded tiles, else a new tile
            const unsigned fw = lane < NS ? vfw[lane] : 0u;
            const unsigned freshm = __ballot_sync(FULL, (fw >> 16) < (fw & 0xffffu));
            const unsigned pfm = __ballot_sync(FULL, lane < NPF && vpfst[lane] == 2);
            const unsigned endm = __ballot_sync(FULL, lane < NPF && vpfst[lane] == 3);
            // every control decision must be warp-uniform (the helpers are warp-collective): shared
            // words that other warps change are read once, by lane 0, and broadcast
            const unsigned freem = __shfl_sync(FULL, lane == 0 ? *vfree : 0u, 0);
            const bool can_claim = pfm && freem;
            int got = 0;
            unsigned fm = freshm;
            for (int tries = 0; tries < 3 && got < 32 && (fm || can_claim); ++tries) {
                const int sl = fm ? __ffs(fm) - 1 : claim();
                if (sl < 0) break;
                fm &= ~(1u << sl);
                got += take_fresh(sl, 32 - got, got, loc, nf);
            }
            if (!got) {
                if (endm == (NPF == 32 ? FULL : (1u << NPF) - 1u) && freem == ALL) break;   // all done
                __nanosleep(backoff);
                backoff = min(2 * backoff, 2048);
                continue;
            }
            backoff = 64;
            cnt = got;
            s = s0;
        }
        // ---------------- one stage for the batch
        const bool act = lane < cnt;
        const int sl = (int)(loc >> 16), idx = (int)(loc & 0xffffu);
        if (act && s == s0) mbar_wait(&mbar[sl], (uint32_t)(s_wpar[sl] ^ 1));   // the tile's plane has landed
        StageDev sd;
        if (s < p.n_pstages) {
            sd.first = p.pstages[s].first;
            sd.n = p.pstages[s].n;
            sd.T = p.pstages[s].T;
            sd.mc = p.pstages[s].mc;
        } else {
            sd = p.stages[s];
        }
        if (lane == 0 && p.stage_counts) atomicAdd(p.stage_counts + s, (unsigned long long)cnt);
        const bool last = s == N - 1;
        float sum = 0.0f;
        bool pass;
#ifndef FD_PACKED_WORDS
        if (cnt <= (FD_DQ_GROUP < 16 ? FD_DQ_GROUP : 16)) {      // (GL >= 2 needs cnt <= 16)
            // thin batch: GL = 2^lg lanes per window share the stage's stumps (records warp-uniform
            // per stump index); the leaves are added as a tree and the decision certified against
            // its rounding bound (k_common.cuh certify) -- the group leader re-adds them in stump
            // order for near ties and for output scores
            int lg = 1;
            while (lg < 5 && (cnt << (lg + 1)) <= 32) ++lg;
            const int e = lane >> lg;
            const bool gact = e < cnt;
            const uint32_t gloc = __shfl_sync(FULL, loc, e & 31);
            const float gnf = __shfl_sync(FULL, nf, e & 31);
            const int gsl = (int)(gloc >> 16), gidx = (int)(gloc & 0xffffu);
            if (gact && s == s0) mbar_wait(&mbar[gsl], (uint32_t)(s_wpar[gsl] ^ 1));
            const int gb = gsl * PBUF + (gidx / TX) * STEP * TW + (gidx % TX) * STEP;
            const float2 t = sd.mc <= 9 ? dq_group_mc<9>(planes, gb, gnf, p.stumps, sd.first, sd.n, lg, gact, lane)
                                        : dq_group_mc<MAX_CORNERS>(planes, gb, gnf, p.stumps, sd.first, sd.n, lg, gact, lane);
            int dec = certify(t.x, t.y, sd.n, (sd.n + (1 << lg) - 1) / (1 << lg) - 1 + lg, sd.T);
            float gsum = t.x;
            if (gact && (lane & ((1 << lg) - 1)) == 0 && (dec < 0 || (dec == 1 && last) || (DEPTH && dec == 0))) {
                gsum = dq_stage(planes, gb, gnf, grec, sd.first, sd.n, sd.mc);
                dec = gsum >= sd.T ? 1 : 0;
            }
            sum = __shfl_sync(FULL, gsum, (lane << lg) & 31);    // back to one lane per window
            dec = __shfl_sync(FULL, dec, (lane << lg) & 31);
            pass = act && dec == 1;
        } else
#endif
        {
            if (act) {
                const int b = sl * PBUF + (idx / TX) * STEP * TW + (idx % TX) * STEP;
#if FD_JIT_DEEPQ > 0
                if (s < FD_JIT_DEEPQ)
                    sum = jit_deepq(s, planes + b, nf);
                else
#endif
#ifdef FD_PACKED_WORDS
                    sum = eval_stage_packed<STEP>(planes, b, nf, sd.first, sd.n);
#else
                    sum = sd.first + sd.n <= p.n_pstumps ? dq_stage(planes, b, nf, prec, sd.first, sd.n, sd.mc)
                                                         : dq_stage(planes, b, nf, grec, sd.first, sd.n, sd.mc);
#endif
            }
            pass = act && sum >= sd.T;
        }
        if (act && !pass) out.reject(sl, idx, s, sum);
        if (pass && last) out.emit(sl, idx, sum);
        // windows that finish here, and (below) windows handed to k_tail, release their slot
        auto release = [&](bool fin, int fsl) {
            const unsigned fm = __ballot_sync(FULL, fin);
            if (fin) {
                const unsigned peers = __match_any_sync(fm, fsl);
                if (lane == __ffs(peers) - 1) {
                    const int k = __popc(peers);
                    if (atomicSub(&s_alive[fsl], k) == k) {  // the tile's last window: free its slot
                        __threadfence_block();
                        atomicOr(&s_free, 1u << fsl);
                    }
                }
            }
        };
        release(act && (!pass || last), sl);
        const unsigned m = __ballot_sync(FULL, pass && !last);
        if (pass && !last) stg[__popc(m & ((1u << lane) - 1u))] = make_uint2(loc, __float_as_uint(nf));
        __syncwarp();
        cnt = __popc(m);
        if (lane < cnt) {
            const uint2 e = stg[lane];
            loc = e.x;
            nf = __uint_as_float(e.y);
        }
        __syncwarp();
        s += 1;
        if (p.tail_q && cnt > 0 && s >= p.s_tail) {
            // long chains leave the pool: windows entering stage s_tail go to k_tail's queue (one warp
            // per window there), so their tile's slot is not held for the rest of the cascade
            int pos = 0;
            if (lane == 0) pos = (int)atomicAdd(p.tail_count, (unsigned)cnt);
            pos = __shfl_sync(FULL, pos, 0);
            const bool hand = lane < cnt && pos + lane < p.tail_cap;
            const int sl2 = (int)(loc >> 16), idx2 = (int)(loc & 0xffffu);
            if (hand) {
                uint4 q;
                q.x = ((unsigned)s_lvl[sl2] << 8) | (unsigned)s;
                q.y = ((unsigned)(s_wy0[sl2] + idx2 / TX) << 16) | (unsigned)(s_wx0[sl2] + idx2 % TX);
                q.z = __float_as_uint(nf);
                q.w = (unsigned)(s_frame[sl2] - p.frame_base);
                p.tail_q[pos + lane] = q;
            }
            const unsigned hm = __ballot_sync(FULL, hand);
            if (hm) {
                if (lane == 0 && p.stage_counts) atomicAdd(p.stage_counts + s, (unsigned long long)__popc(hm));
                release(hand, sl2);
                const int h = __popc(hm);               // the handed lanes are the lowest ones
                if (lane >= h && lane < cnt) stg[lane - h] = make_uint2(loc, __float_as_uint(nf));
                __syncwarp();
                cnt -= h;
                if (lane < cnt) {
                    const uint2 e = stg[lane];
                    loc = e.x;
                    nf = __uint_as_float(e.y);
                }
                __syncwarp();
            }
        }
    }
}

}  // namespace fdk
