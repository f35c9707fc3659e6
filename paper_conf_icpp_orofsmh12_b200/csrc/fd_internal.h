// fd_internal.h -- shared host/device declarations of the CUDA path (not part of the C ABI).
//
// Data layout in HBM:
//   group workspace (u32 elements), per pyramid level k:
//     ws + lv.ws_off + ((g * 2 + plane) * (H_k + 1) + y) * P_k + x
//   plane 0 = ii (u32), plane 1 = sqii mod 2^32 (u32; exact for every 24x24 window
//   difference, reading R4).  P_k = round_up(W_k + 1, 4) so every row is 16-B aligned for
//   TMA and vector stores.  One 4-D TMA tensor map per level covers {x, y, plane, g}.
//   K1 column-sum scratch (u32), per frame: colbuf + g*col_frame + lv.col_off +
//     (band * 2 + plane) * W_k + x
#pragma once
#ifdef __CUDACC_RTC__
// NVRTC build of the K2 kernel (fd_jit.cpp): no host headers; fixed-width types and an opaque
// tensor-map type of the driver's size and alignment
typedef unsigned char uint8_t;
typedef unsigned short uint16_t;
typedef unsigned int uint32_t;
typedef unsigned long long uint64_t;
typedef int int32_t;
typedef long long int64_t;
typedef struct alignas(64) { unsigned long long opaque[16]; } CUtensorMap;
typedef struct CUstream_st* cudaStream_t;
#include "fd.h"
#else
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/fd.h"
#endif

namespace fdk {

constexpr int WIN = FD_WINDOW;       // 24
constexpr int BAND = 32;             // K1 band height (rows)
constexpr int CHUNK = 128;           // K1 chunk width (ii columns): 32 lanes x 4
constexpr int K1_THREADS = 256;
constexpr int REC_WORDS = 16;        // packed stump record: 16 u32 (64 B)
#define FD_PK_WORDS 5                // f3 compressed record (R13): 3 rects (two 16-bit words each), theta|left, right|nrect
constexpr int MAX_CORNERS = 12;
constexpr int MAX_STEP = 4;

// K2 tile geometry per window step (windows per tile TX x TY; a thread owns WPT windows of a
// column; warps tile the x extent in 32-lane columns).  step 1: 8 warps, 64 x 32 windows,
// 88 x 56 ii values per plane.  (32 x 32-window tiles with 4-warp CTAs, 5 resident per SM, were
// measured 30% slower: the per-tile cost of the deep-stage sequence doubles with the tile count.)
__host__ __device__ constexpr int k2_threads(int) { return 256; }
__host__ __device__ constexpr int k2_tx(int step) { return step <= 3 ? 64 : 32; }
__host__ __device__ constexpr int k2_wpt(int step) { return step == 1 ? 8 : (step == 2 ? 4 : (step == 3 ? 2 : 1)); }
__host__ __device__ constexpr int k2_ty(int step) { return (k2_threads(step) / 32 / (k2_tx(step) / 32)) * k2_wpt(step); }
__host__ __device__ constexpr int tile_w(int step) { return (((k2_tx(step) - 1) * step + WIN + 1) + 3) & ~3; }
__host__ __device__ constexpr int tile_h(int step) { return (k2_ty(step) - 1) * step + WIN + 1; }
__host__ __device__ constexpr int k2_pbuf(int step) { return (tile_w(step) * tile_h(step) + 31) & ~31; }


// k_soft (and the former fused K2) shared memory: the tile's ii plane, then its sqii plane -- which,
// once stage 1 has taken every window's variance from it, holds the stage-1 survivor pool
// (nf f32[NW], window u16[NW]) and the two per-stage lists (u16[2][NW]).
template <int STEP>
struct TileGeo {
    static constexpr int PBUF = k2_pbuf(STEP);                          // ii plane (u32)
    static constexpr int NW = k2_tx(STEP) * k2_ty(STEP);
    static constexpr int CP = NW;                                       // pool capacity (a whole tile)
    static constexpr int QBUF = ((PBUF > NW * 10 / 4 ? PBUF : NW * 10 / 4) + 31) & ~31;
    static constexpr size_t OFF_Q = (size_t)PBUF * 4;
    static constexpr size_t OFF_NF = OFF_Q;                             // pool in the sqii buffer
    static constexpr size_t OFF_LOC = OFF_NF + (size_t)NW * 4;
    static constexpr size_t OFF_LIST = OFF_LOC + (size_t)NW * 2;
    static constexpr size_t OFF_RED = OFF_Q + (size_t)QBUF * 4;
    static constexpr size_t SMEM = OFF_RED + (size_t)k2_threads(STEP) * 8;   // + split-stump partial sums
};

// k_stage1 (K2a): two ii planes (the current tile's and the prefetched next tile's), one sqii
// plane (dead once the variance is taken, so the next tile's sqii lands in it during stages 1-2)
// and the stage-1 survivor list (u16 window index + f32 nf)
template <int STEP>
struct TileGeoA {
    static constexpr int PBUF = k2_pbuf(STEP);
    static constexpr int NW = k2_tx(STEP) * k2_ty(STEP);
    static constexpr size_t OFF_Q = (size_t)2 * PBUF * 4;
    static constexpr size_t OFF_SNF = OFF_Q + (size_t)PBUF * 4;
    static constexpr size_t OFF_SIDX = OFF_SNF + (size_t)NW * 4;
    static constexpr size_t SMEM = OFF_SIDX + (size_t)NW * 2;
};

// f1 (fused tile-local integral + cascade): k_f1 stages the tile's level
// PIXELS (u8, one 3-D TMA box from the group's level images) and builds the tile-local ii and
// sqii planes in shared memory -- the same TW x TH layout the TMA'd global planes have, so the
// stage code (incl. the NVRTC-specialised stages) is shared.  Rectangle sums are differences of
// ii values, hence independent of the integral's origin (exact, reading R4).
__host__ __device__ constexpr int f1_nseg(int ph) { return 256 / ph >= 8 ? 8 : (256 / ph >= 4 ? 4 : (256 / ph >= 2 ? 2 : 1)); }
template <int STEP>
struct TileGeoF {
    static constexpr int TW = tile_w(STEP), TH = tile_h(STEP);
    static constexpr int PW = TW - 1, PH = TH - 1;                      // pixel region of a tile
    static constexpr int U8W = (PW + 15) & ~15;                          // TMA box width (16-B multiple)
    static constexpr int UB = (U8W * PH + 127) & ~127;                   // one u8 staging buffer
    static constexpr int PBUF = k2_pbuf(STEP);
    static constexpr int NW = k2_tx(STEP) * k2_ty(STEP);
    static constexpr int CP = NW;
    static constexpr int QBUF = ((PBUF > NW * 10 / 4 ? PBUF : NW * 10 / 4) + 31) & ~31;
    static constexpr size_t OFF_T = (size_t)2 * UB;                       // ii plane
    static constexpr size_t OFF_Q = OFF_T + (size_t)PBUF * 4;             // sqii plane, then the pool
    static constexpr size_t OFF_NF = OFF_Q;
    static constexpr size_t OFF_LOC = OFF_NF + (size_t)NW * 4;
    static constexpr size_t OFF_LIST = OFF_LOC + (size_t)NW * 2;
    static constexpr size_t OFF_RED = OFF_Q + (size_t)QBUF * 4;          // split-stump partial sums
    static constexpr size_t SMEM = OFF_RED + (size_t)k2_threads(STEP) * 8;
};
#ifndef FD_F1_CTAS
#define FD_F1_CTAS 4                        // k_f1: resident CTAs per SM the launch bounds target
#endif

#ifndef FD_K2D_CTAS
#define FD_K2D_CTAS 8
#endif
#ifndef FD_K2D_THREADS
#define FD_K2D_THREADS 128                  // k_deep1 block size (the NVRTC program may override it)
#endif
constexpr int K2D_THREADS = FD_K2D_THREADS;
constexpr int K2D_RED_MAX = 128;            // split-stump partial-sum space, for any k_deep1 block size
template <int STEP, bool F1 = false>
struct TileGeoD {
    static constexpr int PBUF = k2_pbuf(STEP);
    static constexpr int CP = 512;
    static constexpr size_t OFF_NF = (size_t)PBUF * 4;
    static constexpr size_t OFF_LOC = OFF_NF + (size_t)CP * 4;
    static constexpr size_t OFF_LIST = OFF_LOC + (size_t)CP * 2;
    static constexpr size_t OFF_RED = OFF_LIST + (size_t)2 * CP * 2;     // split-stump partial sums
    static constexpr size_t OFF_U8 = (OFF_RED + (size_t)K2D_RED_MAX * 8 + 127) & ~(size_t)127;   // f1 pixels
    static constexpr size_t SMEM = F1 ? OFF_U8 + (size_t)TileGeoF<STEP>::UB : OFF_U8;
};

// k_deepq (K2b, k_deepq.cuh): one persistent CTA per SM; as many tile slots as fit -- each the
// tile's ii plane (TMA) and its first DQ_CAPF stage-s0 survivors -- and a 32-entry staging row
// per warp
#ifndef FD_DQ_WARPS
#define FD_DQ_WARPS 16
#endif
#ifndef FD_DQ_SLOTS
#define FD_DQ_SLOTS 10
#endif
constexpr int DQ_THREADS = FD_DQ_WARPS * 32;
constexpr int DQ_CAPF = 224;                // survivors per slot kept in shared memory (the rest read from HBM)
constexpr size_t DQ_SMEM_MAX = 225 * 1024;  // dynamic shared memory budget (static: < 1 KB)
__host__ __device__ constexpr size_t dq_slot_bytes(int step) { return (size_t)k2_pbuf(step) * 4 + (size_t)DQ_CAPF * 8; }
__host__ __device__ constexpr int dq_slots(int step, int slots, int warps) {
    return slots < (int)((DQ_SMEM_MAX - (size_t)warps * 256) / dq_slot_bytes(step))
               ? slots
               : (int)((DQ_SMEM_MAX - (size_t)warps * 256) / dq_slot_bytes(step));
}
__host__ __device__ constexpr size_t dq_smem(int step, int slots, int warps) {
    return (size_t)dq_slots(step, slots, warps) * dq_slot_bytes(step) + (size_t)warps * 256;
}
template <int STEP>
struct TileGeoQ {
    static constexpr int NS = dq_slots(STEP, FD_DQ_SLOTS, FD_DQ_WARPS);   // tile slots
    static constexpr int PBUF = k2_pbuf(STEP);
    static constexpr size_t OFF_F = (size_t)NS * PBUF * 4;                 // uint2 [NS][DQ_CAPF] survivors
    static constexpr size_t OFF_STG = OFF_F + (size_t)NS * DQ_CAPF * 8;     // uint2 [warps][32]
    static constexpr size_t SMEM = OFF_STG + (size_t)FD_DQ_WARPS * 32 * 8;
    static_assert(NS >= 1 && NS <= 32 && SMEM == dq_smem(STEP, FD_DQ_SLOTS, FD_DQ_WARPS), "k_deepq layout");
};

struct LevelDev {
    int W, H, P;            // level size, ii pitch (elements)
    int PB;                 // f1: u8 level-image pitch (bytes, 16-B multiple >= P)
    long long u8_off;       // f1: byte offset of the level's block u8[G][H][PB] in the group workspace
    int nx, ny;             // windows along x / y (step aware)
    int band0, nbands;      // K1 bands (per frame)
    int tile0, tiles_x;     // K2 tiles (per frame); tiles_y = ceil(ny / TY)
    int r16;                // llround(f * 65536)  (f < 32768 enforced by the plan)
    int nchunks;            // K1 128-column chunks (ceil(P / 128))
    int k1t0;               // first K1 tile (band x chunk) of the level (per frame)
    long long ws_off;       // u32 elements
    long long col_off;      // u32 elements (per frame): column sums/carries [band][2][W]
    long long row_off;      // u32 elements (per frame): row sums/carries [band][chunk][2][BAND]
    long long cor_off;      // u64 elements (per frame): tile corners [band][chunk][2]
    long long lvl_off;      // bytes (per frame): level image [H][PB] written by K1a, read by K1b
    long long win0;         // first window index of the level within a frame
};

struct PlanDev {
    int n_levels;
    int W, H, pitch, step;
    int bands_per_frame;
    int tiles_per_frame;
    int maxW;
    long long win_per_frame;
    long long col_frame;    // K1 scratch elements per frame
    long long row_frame;    // K1 row-carry elements per frame
    long long cor_frame;    // K1 corner elements (u64) per frame
    long long lvl_frame;    // K1 level-image bytes per frame
    int k1tiles_per_frame;  // K1 tiles (band x chunk) per frame
    long long ws_elems;     // group workspace elements (all levels, all g)
    long long u8_bytes;     // f1 group workspace bytes (level images of G frames)
    int G;                  // frames per group (tensor-map extent)
    int filter;             // K1: 1 = binomial 3x3 filtering stage after scaling (f2)
    int aligned4;           // frames pointer and pitch are 4-byte aligned (word loads of identity levels)
    int aligned16;          // ... 16-byte aligned (staged resampling, k_integral.cu stage_source)
    LevelDev lv[FD_MAX_LEVELS];
};

struct StageDev {
    int first;              // index of first stump record
    int n;                  // stumps in stage
    float T;                // stage threshold
    int mc;                 // largest corner count of the stage's stumps (records are zero-padded)
};

// K2 parameters: passed by value as __grid_constant__.  Tensor maps and the level table live
// in global memory; the parameter block (constant bank 0, <= 32 KB) carries a copy of the first
// n_pstumps stump records so warp-uniform record reads use the uniform datapath.
constexpr int PREC_MAX = 440;               // stump records held in parameter space (27.5 KB)
constexpr int PSTAGE_MAX = 64;              // stage descriptors held in parameter space (1 KB)
struct alignas(16) CascadeParams {
    const CUtensorMap* tmaps;               // [n_levels], 64-B aligned, global
    const LevelDev* lv;                     // [n_levels], global
    int n_levels;
    int tiles_per_frame;
    long long win_per_frame;
    const uint4* stumps;                    // REC_WORDS/4 uint4 per stump (all stumps)
    const StageDev* stages;
    int n_stages;
    int n_pstumps;                          // records [0, n_pstumps) are also in prec
    int g_frames;                           // frames in this group
    int frame_base;                         // global index of the group's first frame
    int total_tiles;
    int lane_min;                           // deep stages with fewer survivors use GL lanes per window
    unsigned int* tile_counter;             // zeroed before launch
    unsigned long long* det_count;
    unsigned long long* det_keys;
    float* det_scores;
    long long det_cap;
    uint8_t* depth;                         // depth mode only
    float* score;
    unsigned long long* stage_counts;       // n_stages + 1, may be null
    int n_pstages;                          // stages [0, n_pstages) are also in pstages
    int tail_n;                             // a batch with <= tail_n windows left goes to the tail queue
    int s0;                                 // first stage of the deep kernels (k_stage1 runs [0, s0), s0 <= 2)
    uint4* tail_q;                          // tail queue (k_tail.cu), may be null
    unsigned int* tail_count;               // entries appended (may exceed tail_cap: the excess stays in K2)
    int tail_cap;
    int s_tail;                             // windows still alive at stage s_tail go to the tail queue
    int split_max;                          // deep stages with <= split_max windows use the split-stump mode
    int f1;                                 // 1: tmaps are u8 level-image maps (k_f1, k_deep1 rebuilds ii)
    uint2* surv;                            // split K2: stage-1 survivors (window index, nf bits)
    uint2* tile_rec;                        // split K2: per tile (offset into surv, count)
    unsigned int* surv_count;
    unsigned int* deep_counter;             // k_deep tile claims
    uint4* tile_list;                       // split K2: tiles with stage-s0 survivors {tile, offset, count, 0} (k_deepq)
    unsigned int* tile_list_count;
    StageDev pstages[PSTAGE_MAX];
    uint4 prec[PREC_MAX * (REC_WORDS / 4)];
};

// Tail queue entry (K2 -> k_tail): x = level(8) | stage(8), y = wyi(16) | wxi(16) (window
// indices in the level's step grid), z = nf bits, w = frame index within the group (32 bit).
constexpr int TAIL_RP = 25;                 // row pitch of a window's ii region staged by k_tail
constexpr int TAIL_REC_WORDS = 4 + MAX_CORNERS;   // SoA tail records: nc, theta, left, right, corners
struct TailParams {
    const uint4* q;
    const unsigned int* count;
    int cap;
    int step;
    const uint32_t* ws;                     // group workspace (ii plane 0 read); null in f1 mode
    const uint8_t* lvl8;                    // f1: group level images (the window's ii is rebuilt)
    const LevelDev* lv;
    const uint32_t* trec;                   // [TAIL_REC_WORDS][ns] corner offsets in TAIL_RP pitch
    int ns;
    int j0, nsm;                            // records of stumps [j0, j0 + nsm) are staged in shared memory
    const StageDev* stages;
    int n_stages;
    int frame_base;
    long long win_per_frame;
    unsigned long long* det_count;
    unsigned long long* det_keys;
    float* det_scores;
    long long det_cap;
    uint8_t* depth;
    float* score;
    unsigned long long* stage_counts;
};

// detection key: frame(24) | level(8) | wy(16) | wx(16)
__host__ __device__ inline unsigned long long det_key(int frame, int level, int wy, int wx) {
    return ((unsigned long long)(unsigned)frame << 40) | ((unsigned long long)(unsigned)level << 32) |
           ((unsigned long long)(unsigned)wy << 16) | (unsigned long long)(unsigned)wx;
}

// ---- launchers (implemented in the .cu files) ----
// K1 scratch for one launch of g_frames frames
struct K1Scratch {
    uint32_t* col;          // g_frames * col_frame
    uint32_t* row;          // g_frames * row_frame
    unsigned long long* cor;// g_frames * cor_frame
    uint8_t* lvl;           // g_frames * lvl_frame (resampled level images, pitch P_k)
};
// K1 marginals: per (band, chunk) tile column sums and row sums of p and p^2
cudaError_t launch_k1_marg(const uint8_t* frames, const PlanDev& plan, int g_frames, const K1Scratch& s,
                           cudaStream_t st);
// K1 carries: exclusive scans of the marginals over bands (columns) and chunks (rows), tile corners
cudaError_t launch_k1_carry(const PlanDev& plan, int g_frames, const K1Scratch& s, cudaStream_t st);
// K1 tiles: internal workspace (u32 ii + u32 sqii mod 2^32)
cudaError_t launch_k1_tiles(const uint8_t* frames, const PlanDev& plan, int g_frames, const K1Scratch& s,
                            uint32_t* ws, cudaStream_t st);
// K1 tiles: canonical fd_integral output (u32 ii, u64 sqii) for n images with one level (f = 1)
cudaError_t launch_k1_tiles_canonical(const uint8_t* img, const PlanDev& plan, int n, const K1Scratch& s,
                                      uint32_t* ii, uint64_t* sqii, int out_pitch, cudaStream_t st);
cudaError_t launch_pyramid(const uint8_t* frames, const PlanDev& plan, int n, uint8_t* levels,
                           long long frame_stride, const long long* lvl_off_host, cudaStream_t st);
// f1: level images of a frame group (u8, level-major, pitch PB) and the fused tile-local kernel
cudaError_t launch_levels(const uint8_t* frames, const PlanDev& plan, int g_frames, uint8_t* out, cudaStream_t st);
cudaError_t launch_f1(const CascadeParams& p, bool depth_mode, int step, cudaStream_t st);
cudaError_t launch_tail(const TailParams& p, bool depth_mode, cudaStream_t st);
// split K2: k_stage1 then k_deep (precompiled kernels; step 1 normally runs the NVRTC ones)
cudaError_t launch_stage1(const CascadeParams& p, bool depth_mode, int step, cudaStream_t st);
cudaError_t launch_deep1(const CascadeParams& p, bool depth_mode, int step, bool f1, cudaStream_t st);
cudaError_t launch_deepq(const CascadeParams& p, bool depth_mode, int step, cudaStream_t st);   // k_deepq.cuh
cudaError_t launch_soft(const CascadeParams& p, bool depth_mode, int step, bool soft, cudaStream_t st);  // k_soft.cu (R8b)
cudaError_t launch_depth_hist(const uint8_t* depth, int n, long long win_per_frame, const long long* d_win0,
                              int n_levels, int n_stages, long long* hist, int max_span, cudaStream_t st);
cudaError_t launch_keys_to_dets(const unsigned long long* keys, const float* scores, long long n,
                                const double* f_levels_dev, int n_stages, fd_detection* out, cudaStream_t st);
cudaError_t sort_pairs(void* tmp, size_t& tmp_bytes, const unsigned long long* kin, unsigned long long* kout,
                       const float* vin, float* vout, long long n, cudaStream_t st);
size_t group_scratch_bytes(long long n);
cudaError_t launch_group_plan(const fd_detection* in, long long n, void* scratch, cudaStream_t st);
cudaError_t launch_group_run(const fd_detection* in, long long n, double thresh, int min_neighbors, void* scratch,
                             fd_detection* out, long long cap, long long* d_total, cudaStream_t st);

}  // namespace fdk
