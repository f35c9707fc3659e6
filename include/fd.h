/*
 * fd.h -- C ABI of the B200-native boosted-cascade face detector.
 *
 * Method: Oro, Fernandez, Segura, Martorell, Hernando, "Accelerating Boosting-based Face
 * Detection on GPUs", ICPP 2012 (PAPER.md; citations "P:Lxxx" = line of PAPER.md).
 * Problem statement: "determine the presence of faces in arbitrary images, along with their
 * locations and dimensions" (abstract).  The pipeline is Fig. 1:
 * scaling -> (filtering) -> integral images -> cascade evaluation -> detections.
 * Readings where the paper is silent are listed in DESIGN.md ("Readings", R1..R13).
 *
 * Conventions common to every entry point
 *   - Every function returns fd_status; FD_OK == 0.  On failure a thread-local message is
 *     available from fd_last_error() (valid until the next call on the same thread).
 *   - d_* pointers are CALLER-OWNED DEVICE memory on the current CUDA device; h_* pointers
 *     are caller-owned host memory (pinned is faster, pageable works).  The library owns
 *     only cascade handles and an internal per-(device, stream) workspace that grows on
 *     demand and is released by fd_release_workspaces() or at process exit.
 *   - stream is a cudaStream_t passed as void* (NULL = legacy default stream).  Work is
 *     stream-ordered; calls that must return a count synchronise `stream` once (noted).
 *   - Frames are 8-bit luma ("only the luminance components"), row-major,
 *     frame-major: byte (i, y, x) at frames[i*H*pitch + y*pitch + x].
 *   - FD_EINVAL: W or H < 24, min_size < 24, scale_factor <= 1, step < 1, pitch < W, n < 1,
 *     more than FD_MAX_LEVELS levels, NULL pointers, bad pitch alignment.
 *     FD_EFORMAT: malformed cascade text.  FD_ECAPACITY: result larger than the caller's
 *     buffer (the required count is still returned).  FD_ECUDA: CUDA error (text in
 *     fd_last_error).  FD_ENOMEM: device or host allocation failed.
 */
#ifndef FD_H
#define FD_H

#ifndef __CUDACC_RTC__ /* the K2 kernel source is also compiled at run time by NVRTC (fd_jit.cpp) */
#include <stddef.h>
#include <stdint.h>
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define FD_ABI_VERSION 3
#define FD_MAX_LEVELS 128
#define FD_WINDOW 24 /* fixed 24x24 sliding window, image scaled instead (Fig. 2) */

typedef enum {
    FD_OK = 0,
    FD_EINVAL = 1,
    FD_EFORMAT = 2,
    FD_ECAPACITY = 3,
    FD_ECUDA = 4,
    FD_ENOMEM = 5
} fd_status;

/* Opaque cascade handle: library-owned, immutable after load, usable from several streams. */
typedef struct fd_cascade_s* fd_cascade;

/* One detection (40 bytes).  Detection output of fd_detect: the window at
 * level-space origin (wx, wy) of pyramid level `level` reached the maximum depth; its
 * original-frame rectangle is the back-projection x = floor(wx*f_k + 1/2),
 * y = floor(wy*f_k + 1/2), w = h = floor(24*f_k + 1/2) ("multiplying the downscaling factor by
 * the normalized dimensions").  score = sum of the last stage (the paper's
 * "detection score"; reading R9); aux = depth (= number of stages).
 * For fd_group output: x,y,w,h = rounded member mean, score = max member score,
 * aux = member count, (level, wx, wy) = those of the cluster's first member. */
typedef struct {
    int32_t frame, level, wx, wy;
    int32_t x, y, w, h;
    float score;
    int32_t aux;
} fd_detection;

/* Pyramid plan (host only).  f[k] = (min_size/24) * s^k by repeated multiplication,
 * w[k] = floor(W/f[k]), h[k] = floor(H/f[k]) while both >= 24 (reading R1). */
typedef struct {
    int32_t n_levels;
    double f[FD_MAX_LEVELS];
    int32_t w[FD_MAX_LEVELS], h[FD_MAX_LEVELS];
    int64_t windows[FD_MAX_LEVELS]; /* (floor((w-24)/step)+1) * (floor((h-24)/step)+1) */
    int64_t total_windows;          /* per frame */
} fd_plan;

/* Parse a cascade in .fdc text (format in DESIGN.md "Cascade format": FDC 1 / window 24 24 /
 * optional "filter none|binomial3" / optional "soft" / optional "compress packed16" / stages N /
 * per stage "stage n T" / per stump "stump r (x y w h wt)*r theta left right").
 * "compress packed16" ("reencoding and combining them into two 16-bit
 * words using simple bitwise operations and masks"; reading R13): every rectangle is stored as two
 * 16-bit words (x | y<<5 | w<<10, h | (wt & 63)<<5) and theta/left/right as IEEE binary16; the
 * values in the text must be exactly representable (else FD_EFORMAT) and the stumps evaluated are
 * the ones decoded from the words.  "filter binomial3" switches on the filtering
 * stage between scaling and the integral images (reading R3b) for
 * fd_detect / fd_detect_depth with this cascade; fd_build_pyramid and fd_integral are unfiltered.
 * "soft" makes it a soft cascade (the paper's future work, ref [32]; SURVEY 8(f)
 * f4, reading R8b): the stage sum is not restarted, T_s thresholds the running sum over every
 * stump so far; depth = stages passed, score = the running sum at exit.  At most 250 stages.
 * Stages of growing size evaluated in order with early rejection;
 * stumps are GentleBoost regression stumps on Haar features.
 * Uploads the packed cascade to the CURRENT device.  text need not be NUL-terminated.
 * Errors: FD_EFORMAT (line number in fd_last_error): rect outside the 24x24 window,
 * weight not an integer in [-16,16], r not in {1,2,3}, NaN/inf theta or leaves, NaN T.
 * Ownership: *out is released with fd_free_cascade. */
fd_status fd_load_cascade(const char* text, size_t len, fd_cascade* out);
fd_status fd_free_cascade(fd_cascade c);
fd_status fd_cascade_info(fd_cascade c, int32_t* n_stages, int32_t* n_stumps);

/* Host-only pyramid geometry for a W x H frame (reading R1). */
fd_status fd_pyramid_plan(int W, int H, int min_size, double scale_factor, int step, fd_plan* out);

/* Scaling stage: every pyramid level of n frames, each sampled from the
 * ORIGINAL frame with exact integer bilinear interpolation (reading R2: centre-aligned
 * (x+1/2)f-1/2 in Q16, 8-bit weights, clamp to edge; identity filter, reading R3).
 * d_levels: per frame sum_k w[k]*h[k] bytes, level-major, each level tight (pitch w[k]):
 * byte (i, k, y, x) at d_levels[i*S + off_k + y*w[k] + x], S = sum_k w[k]h[k],
 * off_k = sum_{j<k} w[j]h[j].  Asynchronous. */
fd_status fd_build_pyramid(const uint8_t* d_frames, int n, int W, int H, int pitch, int min_size,
                           double scale_factor, uint8_t* d_levels, void* stream);

/* Integral image computation of n W x H images:
 * ii[y][x] = sum_{y'<y, x'<x} I (uint32), sqii the same over I^2 (uint64), padded exclusive
 * (H+1) x (W+1) (reading R4).  out_pitch (elements) >= W+1 and a multiple of 4; image i at
 * d_ii + i*(H+1)*out_pitch.  Elements [W+1, out_pitch) of each row are written with the row
 * total.  Asynchronous. */
fd_status fd_integral(const uint8_t* d_img, int n, int W, int H, int pitch, uint32_t* d_ii,
                      uint64_t* d_sqii, int out_pitch, void* stream);

/* Cascade evaluation over every window of every pyramid level of n frames:
 * per window the variance normalisation nf (reading R5), Haar features f = sum wt*R
 * (reading R6), stump leaf ((float)f < theta*nf ? left : right) (R7), fp32 stage sums in
 * stump order with early rejection, pass iff sum >= T (R8).  Windows reaching the maximum
 * depth are detections, written to d_out sorted by (frame, level, wy, wx).
 * capacity = elements of d_out.  *n_out = number of detections (host).  If
 * *n_out > capacity returns FD_ECAPACITY and d_out is unspecified.
 * Synchronises `stream` once (to read the count); the records in d_out are complete when
 * `stream` next completes.
 * Schedules (identical results): default K1 (global ii/sqii) -> k_stage1 ->
 * k_deepq (frame groups of >= 4 frames, uncompressed cascades) or k_deep1 -> k_tail (otherwise,
 * or environment FD_DEEPQ=0); environment FD_F1=1 selects SURVEY 8(f) f1 (k_level -> k_f1 with
 * tile-local integrals in shared memory -> k_deep1<F1> -> k_tail; no global integral image).
 * Frames are processed in groups of up to 128 1080p frames (FD_GROUP_MB workspace budget,
 * default 12 GiB: ~48 GB of device memory over the two pipeline slots at 1080p). */
fd_status fd_detect(fd_cascade c, const uint8_t* d_frames, int n, int W, int H, int pitch,
                    int min_size, double scale_factor, int step, fd_detection* d_out,
                    int64_t capacity, int64_t* n_out, void* stream);

/* fd_detect plus per-stage statistics: d_stage_counts (device, n_stages+1 int64, ADDED to):
 * entry s = number of windows that entered stage s (entry 0 = all windows); entry N =
 * accepted.  Stumps evaluated = sum_s entry[s] * stage_size[s]. */
fd_status fd_detect_ex(fd_cascade c, const uint8_t* d_frames, int n, int W, int H, int pitch,
                       int min_size, double scale_factor, int step, fd_detection* d_out,
                       int64_t capacity, int64_t* n_out, int64_t* d_stage_counts, void* stream);

/* The paper's native output: for every window, the deepest stage reached
 * (d_depth, uint8: number of stages passed, N = face) and the sum of the last evaluated stage
 * (d_score, float).  Layout [frame][level][wy/step][wx/step]; per-frame stride
 * plan.total_windows.  Asynchronous. */
fd_status fd_detect_depth(fd_cascade c, const uint8_t* d_frames, int n, int W, int H, int pitch,
                          int min_size, double scale_factor, int step, uint8_t* d_depth,
                          float* d_score, void* stream);

/* Depth-map analytics (Fig. 7: "the
 * distribution of the deepest stage reached by all GPU threads when evaluating the pixels of a
 * given video frame for each considered scale", aggregated over the frames).  d_depth: the
 * fd_detect_depth output for n frames of W x H (same min_size, scale_factor, step), caller-owned
 * device memory.  d_hist: caller-owned device int64[n_levels][n_stages + 1]; hist[k][d] += the
 * number of windows of level k (over the n frames) whose depth is d (d > n_stages counts into
 * bin n_stages).  The rejection rate of stage s at scale k is hist[k][s] / sum_d hist[k][d].
 * d_hist is overwritten (not accumulated).  Exact integer counts.  Asynchronous.
 * Errors: FD_EINVAL for NULL pointers, n < 1, n_stages < 1 or > 254, and the fd_pyramid_plan
 * argument checks. */
fd_status fd_depth_histogram(const uint8_t* d_depth, int n, int W, int H, int min_size, double scale_factor,
                             int step, int n_stages, int64_t* d_hist, void* stream);

/* End-to-end entry with HOST buffers: copies h_frames to the device, runs fd_detect, copies
 * the detections back to h_out (capacity elements).  Synchronises `stream`.  The frames are
 * copied one frame group at a time on that group's pipeline stream, so the copy of a group
 * overlaps the kernels of the previous one (pinned h_frames make the copies asynchronous). */
fd_status fd_detect_host(fd_cascade c, const uint8_t* h_frames, int n, int W, int H, int pitch,
                         int min_size, double scale_factor, int step, fd_detection* h_out,
                         int64_t capacity, int64_t* n_out, void* stream);

/* Grouping: per frame, repeatedly merge the pair of clusters with the smallest
 * S_eyes (eq. 6) while it is < eyes_thresh (paper: 0.5), members averaged;
 * ties -> lexicographically smallest pair (reading R10).  d_in: n detections sorted by frame
 * (fd_detect order).  Clusters with >= min_neighbors members are written to d_out ordered by
 * (frame, first member).  *n_out (host) = count; FD_ECAPACITY if > capacity.
 * Synchronises `stream` once (to read the count). */
fd_status fd_group(const fd_detection* d_in, int64_t n, double eyes_thresh, int min_neighbors,
                   fd_detection* d_out, int64_t capacity, int64_t* n_out, void* stream);

/* fd_detect + fd_group end to end with HOST buffers (the user-facing e2e call): copies
 * h_frames to the device (group by group, overlapped with the previous group's kernels, as
 * fd_detect_host), detects, groups (eyes_thresh, min_neighbors as fd_group) and copies the
 * grouped detections to h_out.  *n_raw (may be NULL) = detections before grouping.
 * Synchronises `stream`. */
fd_status fd_detect_group_host(fd_cascade c, const uint8_t* h_frames, int n, int W, int H, int pitch,
                               int min_size, double scale_factor, int step, double eyes_thresh,
                               int min_neighbors, fd_detection* h_out, int64_t capacity,
                               int64_t* n_out, int64_t* n_raw, void* stream);

/* Kernel accounting (process-wide, all devices): number of launches of each kernel class
 * since the last fd_profile_reset and, if time_kernels != 0, their summed device time
 * measured with CUDA events recorded on the launching stream around each launch.
 * FD_K_SORT is the CUB radix sort (library code, counted as one call).  Default detection
 * path: K1 is FD_K_COLSUM (k_marg: resampling + per-tile marginals), FD_K_CARRY (k_carry +
 * k_corner) and FD_K_BAND (k_tile: ii / sqii); the cascade kernels are FD_K_CASCADE (k_stage1,
 * k_cascade or k_soft) and FD_K_DEEP (k_deepq or k_deep1).  FD_K_TAIL is k_tail (windows handed
 * over one warp per window).  The f1 schedule (FD_F1=1): FD_K_LEVEL (k_level: the group's level
 * images) and FD_K_CASCADE (k_f1: tile-local integral + stages 1-2).  FD_K_DEPTH_HIST is
 * fd_depth_histogram. */
typedef enum {
    FD_K_COLSUM = 0, FD_K_CARRY = 1, FD_K_BAND = 2, FD_K_CASCADE = 3,
    FD_K_SORT = 4, FD_K_DETS = 5, FD_K_GROUP = 6, FD_K_PYRAMID = 7, FD_K_TAIL = 8,
    FD_K_DEEP = 9, FD_K_DEPTH_HIST = 10, FD_K_LEVEL = 11, FD_K_COUNT = 12
} fd_kernel_kind;
typedef struct {
    int64_t launches[FD_K_COUNT];
    double ms[FD_K_COUNT];
} fd_profile;
fd_status fd_profile_reset(int time_kernels);
/* Waits for the recorded events, then returns the totals. */
fd_status fd_profile_read(fd_profile* out);

/* Release every internal workspace of the current device. */
fd_status fd_release_workspaces(void);

/* Thread-local text of the last error ("" if none). */
const char* fd_last_error(void);
int fd_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FD_H */
