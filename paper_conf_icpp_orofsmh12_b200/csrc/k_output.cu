// k_output.cu -- K3 (deterministic detection order + back-projection) and K4 (GPU grouping).
//
// K3: accepted windows arrive from K2 in arbitrary order as 64-bit keys
// frame|level|wy|wx; a radix sort (CUB) makes the output unique and ordered by
// (frame, level, wy, wx), then each key is back-projected to the original frame:
// "the precise dimensions of the sliding window is determined by multiplying the downscaling
// factor by the normalized dimensions"; rounding half up (reading R9), done
// with explicit __dmul_rn/__dadd_rn so no FMA changes the rounding.
//
// K4: grouping: "two detection windows d_i and d_j overlap whenever
// S_eyes(d_i,d_j) < 0.5 ... an iterative process reduces the initial set of windows by
// progressively averaging those with the highest overlapping", S_eyes = eq. 6.
// One CTA per frame; the greedy closest-pair order of the definition (reading R10) is kept
// exactly by maintaining every cluster's nearest neighbour (ties -> lowest index) and
// taking the lexicographically smallest (S, i, j) each round.  Double precision without FMA.
#include <math_constants.h>

#include <cub/cub.cuh>

#include "fd_internal.h"

namespace fdk {

// ------------------------------------------------------------------------------ K3
cudaError_t sort_pairs(void* tmp, size_t& tmp_bytes, const unsigned long long* kin, unsigned long long* kout,
                       const float* vin, float* vout, long long n, cudaStream_t st) {
    return cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, kin, kout, vin, vout, (int)n, 0, 64, st);
}

__global__ void k_keys_to_dets(const unsigned long long* __restrict__ keys, const float* __restrict__ scores, long long n,
                               const double* __restrict__ f, int n_stages, fd_detection* __restrict__ out) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const unsigned long long key = keys[i];
        fd_detection d;
        d.frame = (int)(key >> 40);
        d.level = (int)((key >> 32) & 0xff);
        d.wy = (int)((key >> 16) & 0xffff);
        d.wx = (int)(key & 0xffff);
        const double fk = f[d.level];
        d.x = (int)floor(__dadd_rn(__dmul_rn((double)d.wx, fk), 0.5));
        d.y = (int)floor(__dadd_rn(__dmul_rn((double)d.wy, fk), 0.5));
        d.w = (int)floor(__dadd_rn(__dmul_rn(24.0, fk), 0.5));
        d.h = d.w;
        d.score = scores[i];
        d.aux = n_stages;
        out[i] = d;
    }
}

cudaError_t launch_keys_to_dets(const unsigned long long* keys, const float* scores, long long n, const double* f,
                                int n_stages, fd_detection* out, cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    const int grid = (int)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096);
    k_keys_to_dets<<<grid, 256, 0, st>>>(keys, scores, n, f, n_stages, out);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------ K4
struct Eyes {
    double lex, ley, rex, rey, d;
};

__device__ __forceinline__ Eyes eyes_of(double mx, double my, double mw, double mh) {
    Eyes e;
    e.lex = __dadd_rn(mx, __dmul_rn(0.3, mw));
    e.ley = __dadd_rn(my, __dmul_rn(0.4, mh));
    e.rex = __dadd_rn(mx, __dmul_rn(0.7, mw));
    e.rey = __dadd_rn(my, __dmul_rn(0.4, mh));
    const double dx = __dsub_rn(e.rex, e.lex), dy = __dsub_rn(e.rey, e.ley);
    e.d = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
    return e;
}

__device__ __forceinline__ double s_eyes(const Eyes& a, const Eyes& b) {
    const double lx = __dsub_rn(a.lex, b.lex), ly = __dsub_rn(a.ley, b.ley);
    const double rx = __dsub_rn(a.rex, b.rex), ry = __dsub_rn(a.rey, b.rey);
    const double dle = __dsqrt_rn(__dadd_rn(__dmul_rn(lx, lx), __dmul_rn(ly, ly)));
    const double dre = __dsqrt_rn(__dadd_rn(__dmul_rn(rx, rx), __dmul_rn(ry, ry)));
    const double m = a.d < b.d ? a.d : b.d;
    return __ddiv_rn(__dadd_rn(dle, dre), m);
}

struct GroupScratch {        // per detection (structure of arrays, length n each)
    long long* sx;
    long long* sy;
    long long* sw;
    long long* sh;
    int* cnt;
    float* smax;
    int* nn;
    double* nnd;
    Eyes* eyes;
};

__device__ __forceinline__ Eyes cluster_eyes(const GroupScratch& g, int i) {
    const double n = (double)g.cnt[i];
    return eyes_of(__ddiv_rn((double)g.sx[i], n), __ddiv_rn((double)g.sy[i], n), __ddiv_rn((double)g.sw[i], n),
                   __ddiv_rn((double)g.sh[i], n));
}

// lexicographic (s, a, b) comparison key packed for reductions
struct PairKey {
    double s;
    int a, b;
};
__device__ __forceinline__ bool key_less(const PairKey& x, const PairKey& y) {
    if (x.s < y.s) return true;
    if (y.s < x.s) return false;
    if (x.a != y.a) return x.a < y.a;
    return x.b < y.b;
}

// nearest active neighbour of cluster i among [0, m) (ties -> lowest index); sequential
__device__ void nn_full(const GroupScratch& g, int m, int i) {
    const Eyes ei = g.eyes[i];
    double best = CUDART_INF;
    int bj = -1;
    for (int j = 0; j < m; ++j) {
        if (j == i || g.cnt[j] == 0) continue;
        const double s = s_eyes(ei, g.eyes[j]);
        if (s < best) {
            best = s;
            bj = j;
        }
    }
    g.nn[i] = bj;
    g.nnd[i] = best;
}

constexpr int GT = 256;
constexpr int GLIST = 2048;     // clusters re-scanned warp-parallel per merge (overflow: per thread)

__device__ PairKey block_min(PairKey v, PairKey* red) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        PairKey w;
        w.s = __shfl_xor_sync(0xffffffffu, v.s, o);
        w.a = __shfl_xor_sync(0xffffffffu, v.a, o);
        w.b = __shfl_xor_sync(0xffffffffu, v.b, o);
        if (key_less(w, v)) v = w;
    }
    __syncthreads();
    if (lane == 0) red[warp] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        PairKey r = red[0];
        for (int w = 1; w < GT / 32; ++w)
            if (key_less(red[w], r)) r = red[w];
        red[0] = r;
    }
    __syncthreads();
    return red[0];
}

// Segments = runs of equal frame in the sorted input. seg_start[s], n_seg on device.
// Only pairs with S_eyes < thresh can ever be merged, so nearest neighbours are kept over those
// pairs only (the greedy order of the definition is unchanged: the global minimum pair is the
// same whenever it is below the threshold, and the loop stops otherwise).  A pair whose left-
// or right-eye coordinate gap alone already forces S_eyes >= thresh is skipped without the
// square roots and the division.
__global__ void __launch_bounds__(GT) k_group(const fd_detection* __restrict__ in, long long n,
                                              const long long* __restrict__ seg_start, const int* __restrict__ n_seg_p,
                                              double thresh, int min_neighbors, GroupScratch gs, int* seg_next,
                                              int* seg_count, fd_detection* __restrict__ tmp) {
    __shared__ PairKey red[GT / 32];
    __shared__ int s_seg;
    __shared__ int s_nlist;
    __shared__ int s_list[GLIST];
    const int n_seg = *n_seg_p;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (;;) {
        __syncthreads();
        if (threadIdx.x == 0) s_seg = atomicAdd(seg_next, 1);
        __syncthreads();
        const int sgi = s_seg;
        if (sgi >= n_seg) break;
        const long long a0 = seg_start[sgi];
        const long long a1 = sgi + 1 < n_seg ? seg_start[sgi + 1] : n;
        const int m = (int)(a1 - a0);
        GroupScratch g = gs;
        g.sx += a0; g.sy += a0; g.sw += a0; g.sh += a0; g.cnt += a0; g.smax += a0;
        g.nn += a0; g.nnd += a0; g.eyes += a0;
        for (int i = threadIdx.x; i < m; i += GT) {
            const fd_detection d = in[a0 + i];
            g.sx[i] = d.x; g.sy[i] = d.y; g.sw[i] = d.w; g.sh[i] = d.h;
            g.cnt[i] = 1;
            g.smax[i] = d.score;
            g.eyes[i] = eyes_of((double)d.x, (double)d.y, (double)d.w, (double)d.h);
        }
        __syncthreads();
        // S_eyes of clusters kk, j, or +inf when a single coordinate gap proves S >= thresh:
        // S = (d_le + d_re)/min(d) >= |gap|/min(d); the 2^-40 margin keeps every skipped pair's
        // rounded S above thresh.
        const double tguard = thresh * (1.0 + 0x1p-40);
        auto dist = [&](int kk, int j) -> double {
            const Eyes& a = g.eyes[kk];
            const Eyes& b = g.eyes[j];
            const double lim = tguard * (a.d < b.d ? a.d : b.d);
            if (fabs(a.lex - b.lex) > lim || fabs(a.ley - b.ley) > lim || fabs(a.rex - b.rex) > lim) return CUDART_INF;
            return s_eyes(a, b);
        };
        // warp-parallel nearest neighbour of cluster kk (lowest index on ties)
        auto warp_nn = [&](int kk) {
            double bs = CUDART_INF;
            int bj = 0x7fffffff;
            for (int j = lane; j < m; j += 32) {
                if (j == kk || g.cnt[j] == 0) continue;
                const double s = dist(kk, j);
                if (s < bs) {        // j increases per lane: first minimum = lowest index
                    bs = s;
                    bj = j;
                }
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                const double os = __shfl_xor_sync(0xffffffffu, bs, o);
                const int oj = __shfl_xor_sync(0xffffffffu, bj, o);
                if (os < bs || (os == bs && oj < bj)) {
                    bs = os;
                    bj = oj;
                }
            }
            if (lane == 0) {
                g.nn[kk] = bj == 0x7fffffff ? -1 : bj;
                g.nnd[kk] = bs;
            }
        };
        for (int i = warp; i < m; i += GT / 32) warp_nn(i);
        __syncthreads();
        for (;;) {
            PairKey best;
            best.s = CUDART_INF;
            best.a = 0x7fffffff;
            best.b = 0x7fffffff;
            for (int i = threadIdx.x; i < m; i += GT) {
                if (g.cnt[i] == 0 || g.nn[i] < 0) continue;
                PairKey c;
                c.s = g.nnd[i];
                c.a = min(i, g.nn[i]);
                c.b = max(i, g.nn[i]);
                if (key_less(c, best)) best = c;
            }
            best = block_min(best, red);
            if (!(best.s < thresh) || best.a == 0x7fffffff) break;
            const int a = best.a, b = best.b;
            if (threadIdx.x == 0) {       // merge b into a (sums, count, max score)
                g.sx[a] += g.sx[b]; g.sy[a] += g.sy[b]; g.sw[a] += g.sw[b]; g.sh[a] += g.sh[b];
                g.cnt[a] += g.cnt[b];
                if (g.smax[b] > g.smax[a]) g.smax[a] = g.smax[b];
                g.cnt[b] = 0;
                g.eyes[a] = cluster_eyes(g, a);
                s_nlist = 0;
            }
            __syncthreads();
            // nearest-neighbour maintenance: clusters whose neighbour was a or b (and a itself)
            // are re-scanned warp-parallel below; every other cluster only compares with the new a.
            for (int kk = threadIdx.x; kk < m; kk += GT) {
                if (g.cnt[kk] == 0) continue;
                const int nk = g.nn[kk];
                if (kk == a || nk == a || nk == b) {
                    const int pos = atomicAdd(&s_nlist, 1);
                    if (pos < GLIST) s_list[pos] = kk;
                    else nn_full(g, m, kk);
                } else {
                    const double s = dist(kk, a);
                    if (s < g.nnd[kk] || (s == g.nnd[kk] && a < nk)) {
                        g.nnd[kk] = s;
                        g.nn[kk] = a;
                    }
                }
            }
            __syncthreads();
            {
                const int nl = min(s_nlist, GLIST);
                for (int e = warp; e < nl; e += GT / 32) warp_nn(s_list[e]);
            }
            __syncthreads();
        }
        // emit clusters in first-member order (thread 0; clusters are few)
        if (threadIdx.x == 0) {
            int q = 0;
            for (int i = 0; i < m; ++i) {
                if (g.cnt[i] == 0 || g.cnt[i] < min_neighbors) continue;
                const fd_detection d0 = in[a0 + i];
                const double nn = (double)g.cnt[i];
                fd_detection o;
                o.frame = d0.frame; o.level = d0.level; o.wx = d0.wx; o.wy = d0.wy;
                o.x = (int)floor(__dadd_rn(__ddiv_rn((double)g.sx[i], nn), 0.5));
                o.y = (int)floor(__dadd_rn(__ddiv_rn((double)g.sy[i], nn), 0.5));
                o.w = (int)floor(__dadd_rn(__ddiv_rn((double)g.sw[i], nn), 0.5));
                o.h = (int)floor(__dadd_rn(__ddiv_rn((double)g.sh[i], nn), 0.5));
                o.score = g.smax[i];
                o.aux = g.cnt[i];
                tmp[a0 + q] = o;
                ++q;
            }
            seg_count[sgi] = q;
        }
    }
}

__global__ void k_seg_starts(const fd_detection* __restrict__ in, long long n, long long* seg_start, int* n_seg) {
    // one block: ordered compaction of the starts of equal-frame runs (n = detections, small)
    __shared__ int wsum[32];
    __shared__ int s_total;
    long long base = 0;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (long long c0 = 0; c0 < n; c0 += blockDim.x) {
        const long long i = c0 + threadIdx.x;
        const bool st = i < n && (i == 0 || in[i].frame != in[i - 1].frame);
        const unsigned m = __ballot_sync(0xffffffffu, st);
        if (lane == 0) wsum[warp] = __popc(m);
        __syncthreads();
        if (threadIdx.x == 0) {
            int acc = 0;
            for (int w = 0; w < nw; ++w) {
                const int t = wsum[w];
                wsum[w] = acc;
                acc += t;
            }
            s_total = acc;
        }
        __syncthreads();
        if (st) seg_start[base + wsum[warp] + __popc(m & ((1u << lane) - 1u))] = i;
        base += s_total;
        __syncthreads();
    }
    if (threadIdx.x == 0) *n_seg = (int)base;
}

__global__ void k_seg_offsets(const int* __restrict__ n_seg_p, const int* __restrict__ seg_count, long long* seg_off,
                              long long* total) {
    if (threadIdx.x != 0) return;
    const int ns = *n_seg_p;
    long long acc = 0;
    for (int s = 0; s < ns; ++s) {
        seg_off[s] = acc;
        acc += seg_count[s];
    }
    *total = acc;
}

__global__ void k_seg_copy(const int* __restrict__ n_seg_p, const long long* __restrict__ seg_start,
                           const int* __restrict__ seg_count, const long long* __restrict__ seg_off,
                           const fd_detection* __restrict__ tmp, fd_detection* __restrict__ out, long long cap) {
    const int ns = *n_seg_p;
    for (int s = blockIdx.x; s < ns; s += gridDim.x) {
        const long long a0 = seg_start[s], o0 = seg_off[s];
        for (int i = threadIdx.x; i < seg_count[s]; i += blockDim.x)
            if (o0 + i < cap) out[o0 + i] = tmp[a0 + i];
    }
}

struct GroupLayout {
    GroupScratch g;
    long long* seg_start;
    int* seg_count;
    long long* seg_off;
    fd_detection* tmp;
    int* misc;                 // [0] n_seg, [1] seg_next
    GroupLayout(void* scratch, long long n) {
        char* p = reinterpret_cast<char*>(scratch);
        auto take = [&](size_t bytes) {
            char* r = p;
            p += (bytes + 255) & ~size_t(255);
            return r;
        };
        const size_t a = (size_t)(n > 0 ? n : 1);
        g.sx = reinterpret_cast<long long*>(take(a * 8));
        g.sy = reinterpret_cast<long long*>(take(a * 8));
        g.sw = reinterpret_cast<long long*>(take(a * 8));
        g.sh = reinterpret_cast<long long*>(take(a * 8));
        g.cnt = reinterpret_cast<int*>(take(a * 4));
        g.smax = reinterpret_cast<float*>(take(a * 4));
        g.nn = reinterpret_cast<int*>(take(a * 4));
        g.nnd = reinterpret_cast<double*>(take(a * 8));
        g.eyes = reinterpret_cast<Eyes*>(take(a * sizeof(Eyes)));
        seg_start = reinterpret_cast<long long*>(take(a * 8));
        seg_count = reinterpret_cast<int*>(take(a * 4));
        seg_off = reinterpret_cast<long long*>(take(a * 8));
        tmp = reinterpret_cast<fd_detection*>(take(a * sizeof(fd_detection)));
        misc = reinterpret_cast<int*>(take(256));
    }
};

size_t group_scratch_bytes(long long n) {
    const size_t a = (size_t)(n > 0 ? n : 1);
    return a * (4 * 8 + 4 + 4 + 4 + 8 + sizeof(Eyes) + 8 + 4 + 8 + sizeof(fd_detection)) + 20 * 256;
}

// phase 1: frame segments (runs of equal frame index)
cudaError_t launch_group_plan(const fd_detection* in, long long n, void* scratch, cudaStream_t st) {
    GroupLayout L(scratch, n);
    cudaError_t e = cudaMemsetAsync(L.misc, 0, 256, st);
    if (e != cudaSuccess || n <= 0) return e;
    k_seg_starts<<<1, 1024, 0, st>>>(in, n, L.seg_start, L.misc);
    return cudaGetLastError();
}

// phase 2: greedy grouping per segment, then ordered compaction into out
cudaError_t launch_group_run(const fd_detection* in, long long n, double thresh, int min_neighbors, void* scratch,
                             fd_detection* out, long long cap, long long* d_total, cudaStream_t st) {
    GroupLayout L(scratch, n);
    if (n <= 0) return cudaMemsetAsync(d_total, 0, sizeof(long long), st);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = (int)(n < (long long)sms * 4 ? n : (long long)sms * 4);
    k_group<<<grid, GT, 0, st>>>(in, n, L.seg_start, L.misc, thresh, min_neighbors, L.g, L.misc + 1, L.seg_count, L.tmp);
    k_seg_offsets<<<1, 32, 0, st>>>(L.misc, L.seg_count, L.seg_off, d_total);
    k_seg_copy<<<grid, 256, 0, st>>>(L.misc, L.seg_start, L.seg_count, L.seg_off, L.tmp, out, cap);
    return cudaGetLastError();
}

}  // namespace fdk
