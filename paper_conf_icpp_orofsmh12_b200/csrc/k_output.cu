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
// One CTA per frame, split into independent components (one warp each); the greedy
// closest-pair order of the definition (reading R10) is kept
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
    int* parent;             // union-find over the frame's detections (frame-local indices)
    int* list;               // members of each independent component, increasing index order
    unsigned long long* box; // per component root: 9 bounds (doubles >= 0 as ordered bit patterns)
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

constexpr int GT = 256;
// Segments = runs of equal frame in the sorted input. seg_start[s], n_seg on device.
// One CTA per segment (frame).  The greedy loop is a chain of dependent merges, so the frame is
// first split into INDEPENDENT components and each component runs its own greedy loop in one
// warp (no block barriers per merge):
//   * a cluster's eyes are the mean of its members' eyes and its d lies between its members'
//     (means of the member rectangles), so every cluster of a component stays inside the
//     bounding boxes of the component's left eyes, right eyes and d values;
//   * for clusters A, B of components P, Q: S_eyes(A, B) >= (gap(LE_P, LE_Q) + gap(RE_P, RE_Q)) /
//     min(dmax_P, dmax_Q) (Euclidean gaps between the boxes); components are merged (union-find)
//     until that bound is >= thresh for every pair (with a margin over rounding), so no pair
//     across components ever merges;
//   * merges in different components commute, and inside a component the greedy order is the
//     definition's: smallest (S, i, j) first (frame-local indices, members kept in increasing
//     order), so the final clusters equal those of the frame-wide greedy loop (reading R10).
// Nearest neighbours are kept over pairs with S_eyes < thresh only (the global minimum pair is
// the same whenever it is below the threshold, and the loop stops otherwise); a pair whose
// left- or right-eye coordinate gap alone forces S_eyes >= thresh skips the square roots.
constexpr int GWARPS = GT / 32;
constexpr int GROOTS = 512;             // components tracked per frame (beyond: one component)
constexpr int GPS = 2048;               // frames with <= GPS detections keep union-find in shared memory
constexpr int GBOX = 256;               // ... and, with <= GBOX components, their eye boxes too

// find with path halving: x's parent becomes its grandparent (an ancestor, so concurrent finds and
// root links stay correct); links only ever change a root's parent (uf_union's CAS)
__device__ __forceinline__ int uf_find(int* parent, int x) {
    for (;;) {
        const int q = *reinterpret_cast<volatile int*>(parent + x);
        if (q == x) return x;
        const int qq = *reinterpret_cast<volatile int*>(parent + q);
        if (qq != q) *reinterpret_cast<volatile int*>(parent + x) = qq;
        x = qq;
    }
}
__device__ __forceinline__ void uf_union(int* parent, int a, int b) {
    for (;;) {
        a = uf_find(parent, a);
        b = uf_find(parent, b);
        if (a == b) return;
        if (a < b) {
            const int t = a;
            a = b;
            b = t;
        }
        if (atomicCAS(parent + a, a, b) == a) return;     // root a under the smaller root b
    }
}
__device__ __forceinline__ unsigned long long dbits(double v) { return (unsigned long long)__double_as_longlong(v); }
__device__ __forceinline__ double bitsd(unsigned long long v) { return __longlong_as_double((long long)v); }
// Euclidean gap between intervals boxes [ax0,ax1]x[ay0,ay1] and [bx0,bx1]x[by0,by1]
__device__ __forceinline__ double box_gap(double ax0, double ax1, double ay0, double ay1, double bx0, double bx1,
                                          double by0, double by1) {
    const double gx = fmax(0.0, fmax(__dsub_rn(bx0, ax1), __dsub_rn(ax0, bx1)));
    const double gy = fmax(0.0, fmax(__dsub_rn(by0, ay1), __dsub_rn(ay0, by1)));
    return __dsqrt_rn(__dadd_rn(__dmul_rn(gx, gx), __dmul_rn(gy, gy)));
}
// true when no cluster inside box a can ever reach S_eyes < thresh with one inside box b
// (1e-6 absolute / relative margins over the rounding of cluster means, eyes and d)
__device__ __forceinline__ bool independent(double gl, double gr, double da, double db, double thresh) {
    return __dsub_rn(__dadd_rn(gl, gr), 4e-6) > __dmul_rn(__dmul_rn(thresh, fmin(da, db)), 1.000001);
}

// K4a: one CTA per frame: cluster state, independent components (union-find over the eye-box
// bound), member lists; every component with >= 2 members is appended to the global work list
// comp[] = (frame start a0, list offset, member count).
__global__ void __launch_bounds__(GT) k_group_comp(const fd_detection* __restrict__ in, long long n,
                                                   const long long* __restrict__ seg_start,
                                                   const int* __restrict__ n_seg_p, double thresh, GroupScratch gs,
                                                   int* seg_next, longlong2* comp, int* n_comp) {
    __shared__ int s_seg, s_changed, s_nroots, s_cbase;
    __shared__ int s_roots[GROOTS], s_off[GROOTS], s_cnt[GROOTS];
    __shared__ int s_par[GPS], s_ord[GPS];
    __shared__ unsigned long long s_box[GBOX * 9];
    extern __shared__ float4 s_key[];       // [GPS] dynamic: coarse eye keys
    const int n_seg = *n_seg_p;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (;;) {
        __syncthreads();
        if (tid == 0) s_seg = atomicAdd(seg_next, 1);
        __syncthreads();
        const int sgi = s_seg;
        if (sgi >= n_seg) break;
        const long long a0 = seg_start[sgi];
        const long long a1 = sgi + 1 < n_seg ? seg_start[sgi + 1] : n;
        const int m = (int)(a1 - a0);
        GroupScratch g = gs;
        g.sx += a0; g.sy += a0; g.sw += a0; g.sh += a0; g.cnt += a0; g.smax += a0;
        g.nn += a0; g.nnd += a0; g.eyes += a0; g.parent += a0; g.list += a0; g.box += 9 * a0;
        for (int i = tid; i < m; i += GT) {
            const fd_detection d = in[a0 + i];
            g.sx[i] = d.x; g.sy[i] = d.y; g.sw[i] = d.w; g.sh[i] = d.h;
            g.cnt[i] = 1;
            g.smax[i] = d.score;
            g.eyes[i] = eyes_of((double)d.x, (double)d.y, (double)d.w, (double)d.h);
        }
        const bool fast = m <= GPS;
        int* par = fast ? s_par : g.parent;
        for (int i = tid; i < m; i += GT) {
            par[i] = i;
            if (fast) {
                const Eyes e = g.eyes[i];
                s_key[i] = make_float4((float)e.lex, (float)e.ley, (float)e.rex, (float)e.d);
            }
        }
        __syncthreads();
        __syncthreads();
        // ---- components: singleton pairs first.  A conservative float pre-test on shared-memory
        // keys (lex, ley, rex, d; 1e-2 px slack covers their rounding) skips far pairs; the exact
        // double test follows for the rest
        const float tf = (float)thresh * 1.0001f;
        for (int i = tid; i < m; i += GT) {
            const float4 ki = fast ? s_key[i] : make_float4(0.f, 0.f, 0.f, 0.f);
            const Eyes ei = g.eyes[i];
            for (int j = i + 1; j < m; ++j) {
                if (fast) {
                    const float4 kj = s_key[j];
                    const float lf = __fadd_ru(__fmul_ru(tf, fminf(ki.w, kj.w)), 1e-2f);
                    if (fabsf(ki.x - kj.x) > lf || fabsf(ki.y - kj.y) > lf || fabsf(ki.z - kj.z) > lf) continue;
                }
                const Eyes ej = g.eyes[j];
                const double lim = __dmul_rn(__dmul_rn(thresh, fmin(ei.d, ej.d)), 1.000001) + 4e-6;
                if (fabs(ei.lex - ej.lex) > lim || fabs(ei.ley - ej.ley) > lim || fabs(ei.rex - ej.rex) > lim ||
                    fabs(ei.rey - ej.rey) > lim)
                    continue;
                const double gl = box_gap(ei.lex, ei.lex, ei.ley, ei.ley, ej.lex, ej.lex, ej.ley, ej.ley);
                const double gr = box_gap(ei.rex, ei.rex, ei.rey, ei.rey, ej.rex, ej.rex, ej.rey, ej.rey);
                if (!independent(gl, gr, ei.d, ej.d, thresh)) uf_union(par, i, j);
            }
        }
        // ---- then component boxes, until every pair of components is independent
        bool whole = false;
        for (;;) {
            __syncthreads();
            if (tid == 0) {
                s_changed = 0;
                s_nroots = 0;
            }
            for (int i = tid; i < m; i += GT) par[i] = uf_find(par, i);
            __syncthreads();
            for (int i = tid; i < m; i += GT) {
                if (par[i] != i) continue;
                const int r = atomicAdd(&s_nroots, 1);
                if (r < GROOTS) s_roots[r] = i;
                if (fast) s_ord[i] = r;
                // both candidate boxes (which one is used depends on the final component count)
                unsigned long long* bxs[2] = {g.box + 9 * i, fast && r < GBOX ? s_box + 9 * r : g.box + 9 * i};
#pragma unroll
                for (int t = 0; t < 2; ++t) {
                    unsigned long long* bx = bxs[t];
#pragma unroll
                    for (int c = 0; c < 4; ++c) {
                        bx[2 * c] = dbits(CUDART_INF);
                        bx[2 * c + 1] = 0ull;
                    }
                    bx[8] = 0ull;
                }
            }
            __syncthreads();
            if (s_nroots > GROOTS) {               // too many components to track: one for the frame
                whole = true;
                break;
            }
            // eye boxes: shared-memory atomics when the frame and its component count are small
            const bool sbox = fast && s_nroots <= GBOX;
            auto box_of = [&](int root) -> unsigned long long* {
                return sbox ? s_box + 9 * s_ord[root] : g.box + 9 * root;
            };
            for (int i = tid; i < m; i += GT) {
                const Eyes e = g.eyes[i];
                unsigned long long* bx = box_of(par[i]);
                atomicMin(bx + 0, dbits(e.lex)); atomicMax(bx + 1, dbits(e.lex));
                atomicMin(bx + 2, dbits(e.ley)); atomicMax(bx + 3, dbits(e.ley));
                atomicMin(bx + 4, dbits(e.rex)); atomicMax(bx + 5, dbits(e.rex));
                atomicMin(bx + 6, dbits(e.rey)); atomicMax(bx + 7, dbits(e.rey));
                atomicMax(bx + 8, dbits(e.d));
            }
            __syncthreads();
            const int K = s_nroots;
            const long long npairs = (long long)K * (K - 1) / 2;
            for (long long t = tid; t < npairs; t += GT) {
                // pair index t -> (u, v), u < v
                int u = (int)((sqrt(8.0 * (double)t + 1.0) - 1.0) * 0.5);
                while ((long long)(u + 1) * u / 2 > t) --u;
                while ((long long)(u + 2) * (u + 1) / 2 <= t) ++u;
                const int v = (int)(t - (long long)(u + 1) * u / 2);
                const int ra = s_roots[u + 1], rb = s_roots[v];
                const unsigned long long* A = box_of(ra);
                const unsigned long long* B = box_of(rb);
                const double gl = box_gap(bitsd(A[0]), bitsd(A[1]), bitsd(A[2]), bitsd(A[3]), bitsd(B[0]), bitsd(B[1]),
                                          bitsd(B[2]), bitsd(B[3]));
                const double gr = box_gap(bitsd(A[4]), bitsd(A[5]), bitsd(A[6]), bitsd(A[7]), bitsd(B[4]), bitsd(B[5]),
                                          bitsd(B[6]), bitsd(B[7]));
                if (!independent(gl, gr, bitsd(A[8]), bitsd(B[8]), thresh)) {
                    uf_union(par, ra, rb);
                    s_changed = 1;
                }
            }
            __syncthreads();
            if (!s_changed) break;
        }
        // ---- member lists (increasing index order) per component
        const int K = whole ? 1 : s_nroots;
        if (whole) {
            for (int i = tid; i < m; i += GT) g.list[i] = i;
            if (tid == 0) {
                s_off[0] = 0;
                s_cnt[0] = m;
            }
        } else {
            for (int r = warp; r < K; r += GWARPS) {
                const int root = s_roots[r];
                int c = 0;
                for (int k0 = 0; k0 < m; k0 += 32) {
                    const int i = k0 + lane;
                    c += __popc(__ballot_sync(0xffffffffu, i < m && par[i] == root));
                }
                if (lane == 0) s_cnt[r] = c;
            }
            __syncthreads();
            if (tid == 0) {
                int acc = 0;
                for (int r = 0; r < K; ++r) {
                    s_off[r] = acc;
                    acc += s_cnt[r];
                }
            }
            __syncthreads();
            for (int r = warp; r < K; r += GWARPS) {
                const int root = s_roots[r];
                int c = s_off[r];
                for (int k0 = 0; k0 < m; k0 += 32) {
                    const int i = k0 + lane;
                    const bool in_r = i < m && par[i] == root;
                    const unsigned bm = __ballot_sync(0xffffffffu, in_r);
                    if (in_r) g.list[c + __popc(bm & ((1u << lane) - 1u))] = i;
                    c += __popc(bm);
                }
            }
        }
        __syncthreads();
        __syncthreads();
        // ---- components with >= 2 members -> global work list (one warp each in K4b)
        if (tid == 0) {
            int c = 0;
            for (int r = 0; r < K; ++r) c += s_cnt[r] >= 2;
            s_cbase = c ? atomicAdd(n_comp, c) : 0;
            for (int r = 0, q = s_cbase; r < K; ++r)
                if (s_cnt[r] >= 2) comp[q++] = make_longlong2(a0, ((long long)s_off[r] << 32) | (unsigned)s_cnt[r]);
        }
    }
}

// K4b: the greedy loop of one component per warp, over the components of every frame (the
// merges of different components commute; inside a component the definition's order is kept).
__global__ void __launch_bounds__(GT) k_group_greedy(const longlong2* __restrict__ comp, const int* __restrict__ n_comp,
                                                     double thresh, GroupScratch gs) {
    const int lane = threadIdx.x & 31;
    const double tguard = thresh * (1.0 + 0x1p-40);
    const int nc = *n_comp;
    for (int r = (blockIdx.x * GT + threadIdx.x) >> 5; r < nc; r += (gridDim.x * GT) >> 5) {
        const longlong2 cr = comp[r];
        const long long a0 = cr.x;
        GroupScratch g = gs;
        g.sx += a0; g.sy += a0; g.sw += a0; g.sh += a0; g.cnt += a0; g.smax += a0;
        g.nn += a0; g.nnd += a0; g.eyes += a0; g.parent += a0; g.list += a0; g.box += 9 * a0;
        const int* L = g.list + (int)(cr.y >> 32);
        const int mc = (int)(cr.y & 0xffffffffLL);
        {
            auto dist = [&](const Eyes& a, int j) -> double {
                const Eyes b = g.eyes[j];
                const double lim = tguard * (a.d < b.d ? a.d : b.d);
                if (fabs(a.lex - b.lex) > lim || fabs(a.ley - b.ley) > lim || fabs(a.rex - b.rex) > lim) return CUDART_INF;
                return s_eyes(a, b);
            };
            // nearest neighbour of cluster kk over the component (lowest index on ties)
            auto warp_nn = [&](int kk) {
                const Eyes ek = g.eyes[kk];
                double bs = CUDART_INF;
                int bj = 0x7fffffff;
                for (int q = lane; q < mc; q += 32) {
                    const int j = L[q];
                    if (j == kk || g.cnt[j] == 0) continue;
                    const double s = dist(ek, j);
                    if (s < bs) {
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
            for (int q = lane; q < mc; q += 32) {
                const int i = L[q];
                const Eyes ei = g.eyes[i];
                double bs = CUDART_INF;
                int bj = -1;
                for (int q2 = 0; q2 < mc; ++q2) {
                    const int j = L[q2];
                    if (j == i) continue;
                    const double s = dist(ei, j);
                    if (s < bs) {
                        bs = s;
                        bj = j;
                    }
                }
                g.nn[i] = bj;
                g.nnd[i] = bs;
            }
            __syncwarp();
            for (;;) {
                PairKey best;
                best.s = CUDART_INF;
                best.a = 0x7fffffff;
                best.b = 0x7fffffff;
                for (int q = lane; q < mc; q += 32) {
                    const int i = L[q];
                    if (g.cnt[i] == 0 || g.nn[i] < 0) continue;
                    PairKey c;
                    c.s = g.nnd[i];
                    c.a = min(i, g.nn[i]);
                    c.b = max(i, g.nn[i]);
                    if (key_less(c, best)) best = c;
                }
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    PairKey w;
                    w.s = __shfl_xor_sync(0xffffffffu, best.s, o);
                    w.a = __shfl_xor_sync(0xffffffffu, best.a, o);
                    w.b = __shfl_xor_sync(0xffffffffu, best.b, o);
                    if (key_less(w, best)) best = w;
                }
                if (!(best.s < thresh) || best.a == 0x7fffffff) break;
                const int a = best.a, b = best.b;
                if (lane == 0) {       // merge b into a (sums, count, max score)
                    g.sx[a] += g.sx[b]; g.sy[a] += g.sy[b]; g.sw[a] += g.sw[b]; g.sh[a] += g.sh[b];
                    g.cnt[a] += g.cnt[b];
                    if (g.smax[b] > g.smax[a]) g.smax[a] = g.smax[b];
                    g.cnt[b] = 0;
                    g.eyes[a] = cluster_eyes(g, a);
                }
                __syncwarp();
                // clusters whose neighbour was a or b (and a itself) are re-scanned; every other
                // cluster only compares with the new a
                const Eyes ea = g.eyes[a];
                for (int q0 = 0; q0 < mc; q0 += 32) {
                    const int kk = q0 + lane < mc ? L[q0 + lane] : -1;
                    bool rescan = false;
                    if (kk >= 0 && g.cnt[kk] != 0) {
                        const int nk = g.nn[kk];
                        if (kk == a || nk == a || nk == b) {
                            rescan = true;
                        } else {
                            const double s = dist(ea, kk);
                            if (s < g.nnd[kk] || (s == g.nnd[kk] && a < nk)) {
                                g.nnd[kk] = s;
                                g.nn[kk] = a;
                            }
                        }
                    }
                    unsigned rm = __ballot_sync(0xffffffffu, rescan);
                    __syncwarp();
                    while (rm) {
                        const int t = __ffs(rm) - 1;
                        rm &= rm - 1;
                        warp_nn(L[q0 + t]);
                        __syncwarp();
                    }
                }
            }
        }
    }
}

// K4c: one warp per frame: clusters with >= min_neighbors members, in first-member order.
__global__ void __launch_bounds__(GT) k_group_emit(const fd_detection* __restrict__ in, long long n,
                                                   const long long* __restrict__ seg_start,
                                                   const int* __restrict__ n_seg_p, int min_neighbors, GroupScratch gs,
                                                   int* seg_count, fd_detection* __restrict__ tmp) {
    const int lane = threadIdx.x & 31;
    const int n_seg = *n_seg_p;
    for (int sgi = (blockIdx.x * GT + threadIdx.x) >> 5; sgi < n_seg; sgi += (gridDim.x * GT) >> 5) {
        const long long a0 = seg_start[sgi];
        const long long a1 = sgi + 1 < n_seg ? seg_start[sgi + 1] : n;
        const int m = (int)(a1 - a0);
        GroupScratch g = gs;
        g.sx += a0; g.sy += a0; g.sw += a0; g.sh += a0; g.cnt += a0; g.smax += a0;
        {
            int q = 0;
            for (int k0 = 0; k0 < m; k0 += 32) {
                const int i = k0 + lane;
                const bool keep = i < m && g.cnt[i] != 0 && g.cnt[i] >= min_neighbors;
                const unsigned km = __ballot_sync(0xffffffffu, keep);
                if (keep) {
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
                    tmp[a0 + q + __popc(km & ((1u << lane) - 1u))] = o;
                }
                q += __popc(km);
            }
            if (lane == 0) seg_count[sgi] = q;
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

// ------------------------------------------------------------------------------ depth analytics
// hist[k][d] += #windows of level k with depth d (Fig. 7).  Grid (chunks of the frame's windows,
// frames); a shared histogram per block over the levels its chunk spans.
constexpr int HIST_CHUNK = 4096;
__global__ void __launch_bounds__(256) k_depth_hist(const uint8_t* __restrict__ depth, long long win_per_frame,
                                                    const long long* __restrict__ win0, int n_levels, int nb,
                                                    unsigned long long* __restrict__ hist) {
    extern __shared__ unsigned int sh[];                  // [levels spanned][nb]
    const long long c0 = (long long)blockIdx.x * HIST_CHUNK;
    const long long c1 = min(c0 + HIST_CHUNK, win_per_frame);
    int k0 = 0;
    while (k0 + 1 < n_levels && win0[k0 + 1] <= c0) ++k0;
    int k1 = k0;
    while (k1 + 1 < n_levels && win0[k1 + 1] < c1) ++k1;
    const int span = k1 - k0 + 1;
    for (int i = threadIdx.x; i < span * nb; i += blockDim.x) sh[i] = 0;
    __syncthreads();
    const uint8_t* dp = depth + (long long)blockIdx.y * win_per_frame;
    int k = k0;
    for (long long w = c0 + threadIdx.x; w < c1; w += blockDim.x) {
        while (k > k0 && win0[k] > w) --k;             // w increases per thread: k only moves up
        while (k < k1 && win0[k + 1] <= w) ++k;
        const int d = min((int)dp[w], nb - 1);
        atomicAdd(&sh[(k - k0) * nb + d], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < span * nb; i += blockDim.x)
        if (sh[i]) atomicAdd(hist + (long long)(k0 + i / nb) * nb + i % nb, (unsigned long long)sh[i]);
}

cudaError_t launch_depth_hist(const uint8_t* depth, int n, long long win_per_frame, const long long* d_win0,
                              int n_levels, int n_stages, long long* hist, int max_span, cudaStream_t st) {
    const int nb = n_stages + 1;
    cudaError_t e = cudaMemsetAsync(hist, 0, sizeof(long long) * n_levels * nb, st);
    if (e != cudaSuccess || win_per_frame <= 0) return e;
    const size_t smem = sizeof(unsigned int) * (size_t)max_span * nb;
    e = cudaFuncSetAttribute(k_depth_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const dim3 grid((unsigned)((win_per_frame + HIST_CHUNK - 1) / HIST_CHUNK), (unsigned)n);
    k_depth_hist<<<grid, 256, smem, st>>>(depth, win_per_frame, d_win0, n_levels, nb,
                                          reinterpret_cast<unsigned long long*>(hist));
    return cudaGetLastError();
}

struct GroupLayout {
    GroupScratch g;
    long long* seg_start;
    int* seg_count;
    long long* seg_off;
    fd_detection* tmp;
    longlong2* comp;           // component work list: (frame start, list offset << 32 | members)
    int* misc;                 // [0] n_seg, [1] seg_next, [2] components
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
        g.parent = reinterpret_cast<int*>(take(a * 4));
        g.list = reinterpret_cast<int*>(take(a * 4));
        g.box = reinterpret_cast<unsigned long long*>(take(a * 72));
        seg_start = reinterpret_cast<long long*>(take(a * 8));
        seg_count = reinterpret_cast<int*>(take(a * 4));
        seg_off = reinterpret_cast<long long*>(take(a * 8));
        tmp = reinterpret_cast<fd_detection*>(take(a * sizeof(fd_detection)));
        comp = reinterpret_cast<longlong2*>(take(a * sizeof(longlong2)));
        misc = reinterpret_cast<int*>(take(256));
    }
};

size_t group_scratch_bytes(long long n) {
    const size_t a = (size_t)(n > 0 ? n : 1);
    return a * (4 * 8 + 4 + 4 + 4 + 8 + sizeof(Eyes) + 4 + 4 + 72 + 8 + 4 + 8 + sizeof(fd_detection) + sizeof(longlong2)) +
           24 * 256;
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
    cudaError_t e = cudaFuncSetAttribute(k_group_comp, cudaFuncAttributeMaxDynamicSharedMemorySize, GPS * 16);
    if (e != cudaSuccess) return e;
    k_group_comp<<<grid, GT, GPS * 16, st>>>(in, n, L.seg_start, L.misc, thresh, L.g, L.misc + 1, L.comp, L.misc + 2);
    k_group_greedy<<<sms * 8, GT, 0, st>>>(L.comp, L.misc + 2, thresh, L.g);
    k_group_emit<<<grid, GT, 0, st>>>(in, n, L.seg_start, L.misc, min_neighbors, L.g, L.seg_count, L.tmp);
    k_seg_offsets<<<1, 32, 0, st>>>(L.misc, L.seg_count, L.seg_off, d_total);
    k_seg_copy<<<grid < sms * 4 ? grid : sms * 4, 256, 0, st>>>(L.misc, L.seg_start, L.seg_count, L.seg_off, L.tmp, out, cap);
    return cudaGetLastError();
}

}  // namespace fdk
