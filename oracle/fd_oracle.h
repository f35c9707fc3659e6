/*
 * fd_oracle.h -- plain, slow, obviously-correct CPU oracle for the face-detection hot path
 * of Oro et al., "Accelerating Boosting-based Face Detection on GPUs" (ICPP 2012).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code with
 * the CUDA path (paper_conf_icpp_orofsmh12_b200/) and neither includes the other.
 *
 * Citations are "P:Lxxx" = line of PAPER.md, plus SURVEY.md 8(c) row ids (c1..c10) for
 * the readings taken where the paper is silent.  Every reading is listed in DESIGN.md.
 * Pins: tests/test_oracle.py (brute-force rect sums, closed forms, worked example,
 * all-pass/all-reject cascades, Table I counts, grouping hand cases).
 */
#ifndef FD_ORACLE_H
#define FD_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FDO_MAX_LEVELS 128

typedef struct { int32_t x, y, w, h, wt; } fdo_rect;
typedef struct { int32_t nrect; fdo_rect r[3]; float theta, left, right; } fdo_stump;
typedef struct { int32_t n, first; float T; } fdo_stage;
typedef struct {
    int32_t win_w, win_h, n_stages, n_stumps;
    int32_t filter;          /* 0: identity; 1: binomial 3x3 after scaling (.fdc 'filter binomial3') */
    int32_t soft;            /* 0: stage sums restart at 0 (R8); 1: soft cascade (.fdc 'soft'), the sum runs
                                over all stumps and T_s is a rejection threshold on the running sum (R8b) */
    int32_t packed;          /* 1: '.fdc compress packed16' (f3, reading R13): every stump is stored as two 16-bit
                                words per rectangle + binary16 theta/left/right, and the stumps evaluated are
                                the ones DECODED from those words */
    uint16_t* words;         /* packed16: the compressed stream (per stump: 2 words per rect, theta, left, right) */
    int64_t n_words;
    fdo_stage* stages;
    fdo_stump* stumps;
} fdo_cascade;

/* same 40-byte layout as the product's fd_detection (checked in tests) */
typedef struct {
    int32_t frame, level, wx, wy, x, y, w, h;
    float score;
    int32_t aux;
} fdo_detection;

/* f2: the filtering stage between scaling and the integral image (P:L362-367,
 * taps not given; reading R3b): 3x3 binomial [1 2 1]^T [1 2 1] / 16 with round-half-up
 * ((sum + 8) >> 4) and clamp-to-edge, in place on a W x H (pitch W) level image. */
void fdo_filter_binomial(uint8_t* img, int W, int H);

/* f3 ("reencoding and combining them into two 16-bit words using simple bitwise
 * operations and masks"; reading R13).  Rectangle (x, y, w, h, wt): word 0 = x | y << 5 | w << 10,
 * word 1 = h | (wt & 63) << 5 (wt as 6-bit two's complement).  theta, left, right: IEEE binary16.
 * fdo_half_bits returns -1 if v is not exactly a finite binary16 value. */
int32_t fdo_half_bits(float v);
float fdo_half_value(uint16_t h);
/* stump -> words (2 * nrect + 3); returns the word count, -1 if not representable */
int fdo_pack16(const fdo_stump* s, uint16_t* out);
/* words -> stump (nrect given); returns the words consumed */
int fdo_unpack16(const uint16_t* in, int nrect, fdo_stump* s);
/* the packed stream of a 'compress packed16' cascade (0 words otherwise); returns n_words */
int64_t fdo_cascade_words(const fdo_cascade* c, uint16_t* out, int64_t cap);

/* .fdc text -> cascade (NULL on error, message in err). */
fdo_cascade* fdo_cascade_parse(const char* text, size_t len, char* err, int errlen);
void fdo_cascade_free(fdo_cascade* c);

/* c1: pyramid levels; returns n_levels (0 if none fit, -1 on bad args). */
int fdo_plan(int W, int H, int min_size, double scale, int step, int max_levels,
             double* f, int32_t* Wk, int32_t* Hk, int64_t* nwin);
/* c2: level image (Wk x Hk, tight pitch) sampled from the frame. */
void fdo_resample(const uint8_t* frame, int W, int H, int pitch, double f, int Wk, int Hk, uint8_t* out);
/* c3: ii, sqii of (H+1) x (W+1), tight pitch W+1. */
void fdo_integral(const uint8_t* img, int W, int H, int pitch, uint32_t* ii, uint64_t* sqii);
/* c3/c6: one rectangle sum by the four-corner rule (9 accesses incl. the rect). */
uint32_t fdo_rect_sum(const uint32_t* ii, int ii_pitch, int x, int y, int w, int h);
/* c5: normalisation factor nf of the 24x24 window at (wx, wy). */
float fdo_window_nf(const uint32_t* ii, const uint64_t* sqii, int ii_pitch, int wx, int wy);
/* c6: feature response sum_r wt_r * R_r of the window at (wx, wy). */
int32_t fdo_feature(const uint32_t* ii, int ii_pitch, int wx, int wy, const fdo_rect* r, int nrect);
/* c6 batched for calibration tooling: wins = (wx, wy) pairs. */
void fdo_feature_values(const uint32_t* ii, int ii_pitch, const int32_t* wins, int64_t nw,
                        const fdo_rect* r, int nrect, int32_t* out);
void fdo_window_nf_values(const uint32_t* ii, const uint64_t* sqii, int ii_pitch,
                          const int32_t* wins, int64_t nw, float* out);
/* c7/c8: evaluate one window; returns depth (stages passed); *score = last evaluated stage sum;
 * *near = bit0 stage-sum within 1e-4 of T, bit1 stump near-tie (c11). */
int fdo_eval_window(const fdo_cascade* c, const uint32_t* ii, const uint64_t* sqii, int ii_pitch,
                    int wx, int wy, float* score, int* near);
/* c7/c8 over one level's windows (row-major over (wy/step, wx/step)). */
void fdo_eval_level(const fdo_cascade* c, const uint32_t* ii, const uint64_t* sqii, int Wk, int Hk,
                    int step, uint8_t* depth, float* score, uint8_t* near);

/* Whole path per frame batch (frames u8[n][H][pitch]).
 * fdo_detect: c1..c9; detections sorted (frame, level, wy, wx); returns total count (writes
 * at most cap); *n_near = windows flagged near-threshold.  nthreads: host threads. */
int64_t fdo_detect(const fdo_cascade* c, const uint8_t* frames, int n, int W, int H, int pitch,
                   int min_size, double scale, int step, int nthreads,
                   fdo_detection* out, int64_t cap, int64_t* n_near);
/* per-window depth/score/near maps, layout [frame][level][wy/step][wx/step]. */
int fdo_detect_depth(const fdo_cascade* c, const uint8_t* frames, int n, int W, int H, int pitch,
                     int min_size, double scale, int step, int nthreads,
                     uint8_t* depth, float* score, uint8_t* near);
/* c10: greedy S_eyes grouping (eq. 6).  Input sorted by frame. Returns count. */
int64_t fdo_group(const fdo_detection* in, int64_t n, double eyes_thresh, int min_neighbors,
                  fdo_detection* out, int64_t cap);
/* eq. 6 between two rectangles given as doubles (for pins). */
double fdo_s_eyes(double ax, double ay, double aw, double ah, double bx, double by, double bw, double bh);

#ifdef __cplusplus
}
#endif
#endif
