// k_deepq.cuh -- K2b, the deep stages (s0 .. N-1) as warp-autonomous batches over a per-SM pool of
// tiles (included by k_cascade.cu; also compiled by NVRTC with the cascade's specialised stages).
//
// The paper evaluates the deeper stages in the thread that owns the window, so warps empty out as
// windows are rejected (the divergence problem; Fig. 7's rejection profile,
// P:L1311-1325).  k_stage1 leaves ~1.7% of the windows alive after stage 2, ~70 per tile that has
// any.  Here one persistent CTA per SM keeps NS tiles' ii planes in shared memory (TMA, one
// mbarrier per slot) and every warp works on its own batch of up to 32 windows, one lane per
// window, all at the same stage s so the stump records stay warp-uniform (parameter bank):
//   * after a stage the warp compacts its survivors (ballot + rank), tops them up from the ring of
//     stage s+1, and keeps going while the batch is at least DQ_KEEP windows; a thinner batch is
//     parked in that ring when fuller work exists -- a ring holding >= 32 windows (deepest
//     first), fresh windows of a loaded tile, or a new tile (claimed into a free slot); with
//     nothing fuller it continues, and an idle warp takes the deepest non-empty ring;
//   * no CTA barrier and no lock after the start: the rings are multi-producer multi-consumer
//     (head / tail reserved with CAS, a sequence word per cell publishes and frees it), fresh
//     windows are taken with a CAS on the slot's (taken | n) word, slots and prefetched tile-list
//     entries with atomics, so a tile's slowest window never holds up the others;
//   * a slot is reloaded once every window of its tile has finished (per-slot alive count).
// Windows of different tiles share a batch (each lane addresses its own slot's plane).  Decisions,
// scores and outputs are the definition's: lane-per-window sequential fp32 sums (oracle c7/c8).
#pragma once

namespace fdk {

#ifndef FD_DQ_NPF
#define FD_DQ_NPF 4             // tile-list entries prefetched per CTA
#endif
#ifndef FD_DQ_KEEP
#define FD_DQ_KEEP 24           // a batch thinner than this is parked when fuller work exists
#endif

template <int STEP, bool DEPTH>
__global__ void __launch_bounds__(DQ_THREADS, 1) k_deepq(const __grid_constant__ CascadeParams p) {
    using G = TileGeoQ<STEP>;
    constexpr int TX = k2_tx(STEP), TW = tile_w(STEP), PBUF = G::PBUF, PLANE = tile_w(STEP) * tile_h(STEP);
    constexpr int NS = G::NS, NQ = DQ_NQ, QC = DQ_QC, NPF = FD_DQ_NPF;
    constexpr unsigned ALL = (NS == 32) ? 0xffffffffu : ((1u << NS) - 1u);
    constexpr unsigned FULL = 0xffffffffu;
    static_assert(NQ <= 32 && NPF <= 32 && (QC & (QC - 1)) == 0, "one lane per ring / entry; QC a power of two");
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    const uint32_t* planes = reinterpret_cast<const uint32_t*>(smem_raw);
    volatile uint2* ent = reinterpret_cast<volatile uint2*>(smem_raw + G::OFF_Q);     // [NQ][QC] {loc, nf bits}
    volatile int* seq = reinterpret_cast<volatile int*>(smem_raw + G::OFF_SEQ);        // [NQ][QC]
    uint2* stg = reinterpret_cast<uint2*>(smem_raw + G::OFF_STG) + (threadIdx.x >> 5) * 32;   // this warp's
    __shared__ __align__(8) uint64_t mbar[NS];
    __shared__ int s_frame[NS], s_lvl[NS], s_wx0[NS], s_wy0[NS];
    __shared__ int s_alive[NS];             // windows of the slot's tile not finished yet
    __shared__ unsigned s_fw[NS];           // fresh windows: taken << 16 | n (taken == n: none left)
    __shared__ int s_foff[NS];              // the tile's survivors: p.surv[foff, foff + n)
    __shared__ int s_wpar[NS];              // mbarrier parity of the slot's current load
    __shared__ unsigned s_free;
    __shared__ int s_head[NQ], s_tail[NQ];  // ring q: windows entering stage s0 + 1 + q
    __shared__ int s_pfst[NPF];             // prefetched tile-list entries: 0 filling, 1 owned, 2 ready, 3 none left
    __shared__ int4 s_pf0[NPF], s_pf1[NPF]; // {tile, off, n, -}, {g, k, wx0, wy0}
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int N = p.n_stages, s0 = p.s0;
    const ParamRec prec{p};
    const GlobalRec grec{p.stumps};
    const WinOut<STEP, DEPTH> out{p, s_frame, s_lvl, s_wx0, s_wy0};
    volatile int* vhead = s_head;
    volatile int* vtail = s_tail;
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
    if (tid < NQ) s_head[tid] = s_tail[tid] = 0;
    for (int c = tid; c < NQ * QC; c += DQ_THREADS) seq[c] = c & (QC - 1);   // cell free for lap 0
    if (tid < NPF) s_pfst[tid] = 0;
    __syncthreads();
    if (lane == 0 && warp < NPF) refill(warp);

    // ring j: pop up to k (at least kmin) entries into lanes [dst, dst + got); warp-uniform result
    auto ring_pop = [&](int j, int k, int kmin, int dst, uint32_t& loc, float& nf) -> int {
        int base = 0, got = 0;
        if (lane == 0) {
            for (;;) {
                const int hd = vhead[j], tl = vtail[j];
                const int t = min(k, tl - hd);
                if (t < kmin || t <= 0) break;
                if (atomicCAS(&s_head[j], hd, hd + t) == hd) {
                    base = hd;
                    got = t;
                    break;
                }
            }
        }
        got = __shfl_sync(FULL, got, 0);
        base = __shfl_sync(FULL, base, 0);
        if (lane >= dst && lane < dst + got) {
            const int pos = base + lane - dst, cell = j * QC + (pos & (QC - 1));
            while (seq[cell] != pos + 1) {}                  // the pusher's entry has landed
            __threadfence_block();
            const uint2 e = make_uint2(ent[cell].x, ent[cell].y);
            loc = e.x;
            nf = __uint_as_float(e.y);
            __threadfence_block();
            seq[cell] = pos + QC;                            // free for the next lap
        }
        return got;
    };
    // ring j: push lanes [0, c); false (nothing written) when the ring has no room
    auto ring_push = [&](int j, int c, uint32_t loc, float nf) -> bool {
        int base = -1;
        if (lane == 0) {
            for (;;) {
                const int tl = vtail[j], hd = vhead[j];
                if (tl - hd + c > QC) break;
                if (atomicCAS(&s_tail[j], tl, tl + c) == tl) {
                    base = tl;
                    break;
                }
            }
        }
        base = __shfl_sync(FULL, base, 0);
        if (base < 0) return false;
        if (lane < c) {
            const int pos = base + lane, cell = j * QC + (pos & (QC - 1));
            while (seq[cell] != pos) {}                      // the previous lap's reader is done
            ent[cell].x = loc;
            ent[cell].y = __float_as_uint(nf);
            __threadfence_block();
            seq[cell] = pos + 1;
        }
        return true;
    };
    // fresh windows of slot sl into lanes [dst, dst + got), at most k; warp-uniform result
    auto take_fresh = [&](int sl, int k, int dst, uint32_t& loc, int& fidx) -> int {
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
            loc = (uint32_t)sl << 16;
            fidx = *reinterpret_cast<volatile int*>(&s_foff[sl]) + t0 + (lane - dst);
        }
        return got;
    };
    // claim a prefetched tile into a free slot (TMA of its ii plane); the slot index or -1
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
                    __threadfence_block();
                    vfw[sl] = (unsigned)a.z;                 // publish: 0 taken of n
                    refill(pf);
                }
            }
        }
        return __shfl_sync(FULL, sl, 0);
    };

    int cnt = 0, s = s0;          // this warp's batch: lanes [0, cnt) hold windows entering stage s
    uint32_t loc = 0;             // slot << 16 | window index within the slot's tile
    float nf = 1.0f;
    int backoff = 64;
    for (;;) {
        if (cnt < 32) {
            // ---------------- scheduling: every lane reads one ring / slot / prefetch entry
            const int qn = lane < NQ ? vtail[lane] - vhead[lane] : 0;
            const unsigned fullm = __ballot_sync(FULL, qn >= 32);
            const unsigned nonem = __ballot_sync(FULL, qn > 0);
            const unsigned fw = lane < NS ? vfw[lane] : 0u;
            const unsigned freshm = __ballot_sync(FULL, (fw >> 16) < (fw & 0xffffu));
            const unsigned pfm = __ballot_sync(FULL, lane < NPF && vpfst[lane] == 2);
            const unsigned endm = __ballot_sync(FULL, lane < NPF && vpfst[lane] == 3);
            // every control decision below must be warp-uniform (the helpers are warp-collective):
            // shared words that other warps change are read once, by lane 0, and broadcast
            const unsigned freem = __shfl_sync(FULL, lane == 0 ? *vfree : 0u, 0);
            const bool can_claim = pfm && freem;
            const int qi = s - (s0 + 1);
            const bool ring_s = cnt > 0 && qi >= 0 && qi < NQ;
            if (ring_s && (nonem >> qi) & 1u) cnt += ring_pop(qi, 32 - cnt, 1, cnt, loc, nf);
            if (ring_s && cnt < FD_DQ_KEEP && ((fullm & ~(1u << qi)) || freshm || can_claim)) {
                if (ring_push(qi, cnt, loc, nf)) cnt = 0;      // parked; take fuller work
            }
            int fidx = -1;
            if (cnt == 0) {
                int got = 0;
                if (fullm) {
                    const int j = 31 - __clz(fullm);
                    got = ring_pop(j, 32, 32, 0, loc, nf);
                    s = s0 + 1 + j;
                }
                if (!got && (freshm || can_claim)) {
                    unsigned fm = freshm;
                    for (int tries = 0; tries < 3 && got < 32; ++tries) {
                        int sl = fm ? __ffs(fm) - 1 : claim();
                        if (sl < 0) break;
                        fm &= ~(1u << sl);
                        got += take_fresh(sl, 32 - got, got, loc, fidx);
                        if (!fm && got < 32 && !can_claim) break;
                    }
                    s = s0;
                }
                if (!got && nonem) {
                    const int j = 31 - __clz(nonem);
                    got = ring_pop(j, 32, 1, 0, loc, nf);
                    s = s0 + 1 + j;
                }
                if (!got) {
                    const unsigned fr2 = __shfl_sync(FULL, lane == 0 ? *vfree : 0u, 0);
                    if (endm == (NPF == 32 ? FULL : (1u << NPF) - 1u) && fr2 == ALL && !nonem) break;   // all done
                    __nanosleep(backoff);
                    backoff = min(2 * backoff, 2048);
                    continue;
                }
                backoff = 64;
                cnt = got;
            }
            if (fidx >= 0) {                               // fresh window: index and nf from k_stage1's list
                const uint2 v = p.surv[fidx];
                loc |= v.x;
                nf = __uint_as_float(v.y);
            }
        }
        // ---------------- one stage for the batch, lane per window
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
        float sum = 0.0f;
        if (act) {
            const int b = sl * PBUF + (idx / TX) * STEP * TW + (idx % TX) * STEP;
#if FD_JIT_DEEP > 0
            if (s < FD_JIT_DEEP)
                sum = jit_deep(s, planes + b, nf);
            else
#endif
#ifdef FD_PACKED_WORDS
                sum = eval_stage_packed<STEP>(planes, b, nf, sd.first, sd.n);
#else
                sum = sd.first + sd.n <= p.n_pstumps ? eval_stage(planes, b, nf, prec, sd.first, sd.n, sd.mc)
                                                     : eval_stage(planes, b, nf, grec, sd.first, sd.n, sd.mc);
#endif
        }
        const bool pass = act && sum >= sd.T;
        const bool last = s == N - 1;
        if (act && !pass) out.reject(sl, idx, s, sum);
        if (pass && last) out.emit(sl, idx, sum);
        const bool fin = act && (!pass || last);
        const unsigned finm = __ballot_sync(FULL, fin);
        if (fin) {
            // per-slot alive counts; the window that finishes a tile frees its slot
            const unsigned peers = __match_any_sync(finm, sl);
            if (lane == __ffs(peers) - 1) {
                const int k = __popc(peers);
                if (atomicSub(&s_alive[sl], k) == k) {
                    __threadfence_block();
                    atomicOr(&s_free, 1u << sl);
                }
            }
        }
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
    }
}

}  // namespace fdk
