/*
 * fd_oracle.c -- plain CPU oracle (TEST INFRASTRUCTURE; see fd_oracle.h header).
 *
 * Written from PAPER.md and the readings in SURVEY.md 8(c) / DESIGN.md "Readings".
 * No blocking, fusion or reordering: each step is the definition written out, in the
 * paper's order (scale -> integral image -> per-window cascade walk, Fig. 1 P:L292-314,
 * P:L316-408).  Compile with -O2 -ffp-contract=off -fno-fast-math (no FMA contraction,
 * IEEE sqrtf), which the build enforces.
 */
#include "fd_oracle.h"

#include <ctype.h>
#include <math.h>
#include <pthread.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#define WIN 24
#define WIN_AREA 576

/* ------------------------------------------------------------------------------------ */
/* .fdc parser (the oracle's own; the CUDA library has a separate one)                   */
/* ------------------------------------------------------------------------------------ */

typedef struct { const char* p; const char* end; int line; } cursor_t;

static int next_line(cursor_t* c, char* buf, int cap) {
    for (;;) {
        if (c->p >= c->end) return 0;
        const char* q = c->p;
        while (q < c->end && *q != '\n') ++q;
        int n = (int)(q - c->p);
        if (n >= cap) n = cap - 1;
        memcpy(buf, c->p, (size_t)n);
        buf[n] = 0;
        c->p = q < c->end ? q + 1 : q;
        c->line++;
        char* s = buf;
        while (*s && isspace((unsigned char)*s)) ++s;
        if (*s == 0 || *s == '#') continue;
        return 1;
    }
}

static int tok_long(char** s, long* v) {
    while (**s && isspace((unsigned char)**s)) ++*s;
    if (!**s) return 0;
    char* e;
    *v = strtol(*s, &e, 10);
    if (e == *s || (*e && !isspace((unsigned char)*e))) return 0;
    *s = e;
    return 1;
}

static int tok_float(char** s, float* v, int allow_inf) {
    while (**s && isspace((unsigned char)**s)) ++*s;
    if (!**s) return 0;
    char* e;
    *v = strtof(*s, &e);
    if (e == *s || (*e && !isspace((unsigned char)*e))) return 0;
    if (isnan(*v)) return 0;
    if (!allow_inf && isinf(*v)) return 0;
    *s = e;
    return 1;
}

static int tok_word(char** s, const char* w) {
    while (**s && isspace((unsigned char)**s)) ++*s;
    size_t n = strlen(w);
    if (strncmp(*s, w, n) != 0) return 0;
    if ((*s)[n] && !isspace((unsigned char)(*s)[n])) return 0;
    *s += n;
    return 1;
}

static int at_end(char* s) {
    while (*s && isspace((unsigned char)*s)) ++s;
    return *s == 0;
}

void fdo_cascade_free(fdo_cascade* c) {
    if (!c) return;
    free(c->stages);
    free(c->stumps);
    free(c->words);
    free(c);
}

/* ------------------------------------------------------------------------------------ */
/* f3: compressed feature records (reading R13)                              */
/* ------------------------------------------------------------------------------------ */

/* IEEE binary16 value of h: (-1)^s * 2^(e-15) * (1 + m/1024) for 1 <= e <= 30,
 * (-1)^s * 2^-14 * (m/1024) for e = 0 (subnormals and zero); e = 31 is inf / NaN. */
float fdo_half_value(uint16_t h) {
    const int sgn = h >> 15, e = (h >> 10) & 31, m = h & 1023;
    double v;
    if (e == 31) v = m ? NAN : INFINITY;
    else if (e == 0) v = ldexp((double)m, -24);
    else v = ldexp(1024.0 + (double)m, e - 25);
    return (float)(sgn ? -v : v);
}

/* binary16 bits of v if v is exactly a finite binary16 value, else -1: search the exponent whose
 * grid contains v (plain definition, no conversion intrinsics) */
int32_t fdo_half_bits(float v) {
    if (!isfinite(v)) return -1;
    const int sgn = signbit(v) ? 1 : 0;
    const double a = fabs((double)v);
    if (a == 0.0) return sgn << 15;
    for (int e = 0; e <= 30; ++e) {
        /* values of exponent field e: subnormal m * 2^-24 (e = 0), else (1024 + m) * 2^(e-25) */
        const double scale = ldexp(1.0, e == 0 ? -24 : e - 25);
        const double q = a / scale;                    /* exact: scale is a power of two */
        const double lo = e == 0 ? 1.0 : 1024.0, hi = e == 0 ? 1023.0 : 2047.0;
        if (q >= lo && q <= hi && q == floor(q)) return (sgn << 15) | (e << 10) | ((int)q - (e == 0 ? 0 : 1024));
    }
    return -1;
}

int fdo_pack16(const fdo_stump* s, uint16_t* out) {
    int n = 0;
    for (int r = 0; r < s->nrect; ++r) {
        const fdo_rect* q = &s->r[r];
        if (q->x < 0 || q->x > 31 || q->y < 0 || q->y > 31 || q->w < 0 || q->w > 31 || q->h < 0 || q->h > 31 ||
            q->wt < -32 || q->wt > 31)
            return -1;
        out[n++] = (uint16_t)(q->x | (q->y << 5) | (q->w << 10));
        out[n++] = (uint16_t)(q->h | ((q->wt & 63) << 5));
    }
    const int32_t t = fdo_half_bits(s->theta), l = fdo_half_bits(s->left), rr = fdo_half_bits(s->right);
    if (t < 0 || l < 0 || rr < 0) return -1;
    out[n++] = (uint16_t)t;
    out[n++] = (uint16_t)l;
    out[n++] = (uint16_t)rr;
    return n;
}

int fdo_unpack16(const uint16_t* in, int nrect, fdo_stump* s) {
    int n = 0;
    memset(s, 0, sizeof *s);
    s->nrect = nrect;
    for (int r = 0; r < nrect; ++r) {
        const uint16_t a = in[n++], b = in[n++];
        s->r[r].x = a & 31;
        s->r[r].y = (a >> 5) & 31;
        s->r[r].w = (a >> 10) & 31;
        s->r[r].h = b & 31;
        const int wt = (b >> 5) & 63;
        s->r[r].wt = wt >= 32 ? wt - 64 : wt;          /* 6-bit two's complement */
    }
    s->theta = fdo_half_value(in[n++]);
    s->left = fdo_half_value(in[n++]);
    s->right = fdo_half_value(in[n++]);
    return n;
}

int64_t fdo_cascade_words(const fdo_cascade* c, uint16_t* out, int64_t cap) {
    if (!c->packed) return 0;
    if (out)
        for (int64_t i = 0; i < c->n_words && i < cap; ++i) out[i] = c->words[i];
    return c->n_words;
}

#define PERR(...) do { if (err && errlen > 0) snprintf(err, (size_t)errlen, __VA_ARGS__); goto fail; } while (0)

fdo_cascade* fdo_cascade_parse(const char* text, size_t len, char* err, int errlen) {
    cursor_t cur = {text, text + len, 0};
    char line[4096];
    char* s;
    long v, ww, wh;
    fdo_cascade* c = (fdo_cascade*)calloc(1, sizeof(fdo_cascade));
    if (!c) return NULL;
    if (!next_line(&cur, line, sizeof line)) PERR("line %d: empty cascade", cur.line);
    s = line;
    if (!tok_word(&s, "FDC") || !tok_long(&s, &v) || v != 1 || !at_end(s)) PERR("line %d: expected 'FDC 1'", cur.line);
    if (!next_line(&cur, line, sizeof line)) PERR("line %d: missing window", cur.line);
    s = line;
    if (!tok_word(&s, "window") || !tok_long(&s, &ww) || !tok_long(&s, &wh) || !at_end(s))
        PERR("line %d: expected 'window 24 24'", cur.line);
    if (ww != WIN || wh != WIN) PERR("line %d: window must be 24 24", cur.line);
    c->win_w = (int32_t)ww;
    c->win_h = (int32_t)wh;
    if (!next_line(&cur, line, sizeof line)) PERR("line %d: missing stages", cur.line);
    s = line;
    if (tok_word(&s, "filter")) {         /* optional: 'filter none' | 'filter binomial3' */
        if (tok_word(&s, "binomial3") && at_end(s))
            c->filter = 1;
        else if (tok_word(&s, "none") && at_end(s))
            c->filter = 0;
        else
            PERR("line %d: expected 'filter none' or 'filter binomial3'", cur.line);
        if (!next_line(&cur, line, sizeof line)) PERR("line %d: missing stages", cur.line);
        s = line;
    } else {
        s = line;
    }
    if (tok_word(&s, "soft")) {           /* optional: soft cascade (f4, reading R8b) */
        if (!at_end(s)) PERR("line %d: expected 'soft'", cur.line);
        c->soft = 1;
        if (!next_line(&cur, line, sizeof line)) PERR("line %d: missing stages", cur.line);
        s = line;
    } else {
        s = line;
    }
    if (tok_word(&s, "compress")) {       /* optional: compressed records (f3, reading R13) */
        if (!tok_word(&s, "packed16") || !at_end(s)) PERR("line %d: expected 'compress packed16'", cur.line);
        c->packed = 1;
        if (!next_line(&cur, line, sizeof line)) PERR("line %d: missing stages", cur.line);
        s = line;
    } else {
        s = line;
    }
    if (!tok_word(&s, "stages") || !tok_long(&s, &v) || !at_end(s) || v < 1 || v > 4096)
        PERR("line %d: expected 'stages N' (1..4096)", cur.line);
    c->n_stages = (int32_t)v;
    c->stages = (fdo_stage*)calloc((size_t)v, sizeof(fdo_stage));
    if (!c->stages) PERR("out of memory");
    int cap = 64;
    c->stumps = (fdo_stump*)malloc(sizeof(fdo_stump) * (size_t)cap);
    if (!c->stumps) PERR("out of memory");
    for (int st = 0; st < c->n_stages; ++st) {
        long n;
        float T;
        if (!next_line(&cur, line, sizeof line)) PERR("line %d: missing stage %d", cur.line, st);
        s = line;
        if (!tok_word(&s, "stage") || !tok_long(&s, &n) || !tok_float(&s, &T, 1) || !at_end(s) || n < 1 || n > 65536)
            PERR("line %d: expected 'stage n T'", cur.line);
        c->stages[st].n = (int32_t)n;
        c->stages[st].first = c->n_stumps;
        c->stages[st].T = T;
        for (long j = 0; j < n; ++j) {
            long nr;
            if (!next_line(&cur, line, sizeof line)) PERR("line %d: missing stump", cur.line);
            s = line;
            if (!tok_word(&s, "stump") || !tok_long(&s, &nr) || nr < 1 || nr > 3)
                PERR("line %d: expected 'stump r ...' with r in 1..3", cur.line);
            if (c->n_stumps == cap) {
                cap *= 2;
                fdo_stump* ns = (fdo_stump*)realloc(c->stumps, sizeof(fdo_stump) * (size_t)cap);
                if (!ns) PERR("out of memory");
                c->stumps = ns;
            }
            fdo_stump* sp = &c->stumps[c->n_stumps];
            memset(sp, 0, sizeof *sp);
            sp->nrect = (int32_t)nr;
            for (long r = 0; r < nr; ++r) {
                long x, y, w, h, wt;
                if (!tok_long(&s, &x) || !tok_long(&s, &y) || !tok_long(&s, &w) || !tok_long(&s, &h) || !tok_long(&s, &wt))
                    PERR("line %d: bad rectangle", cur.line);
                if (x < 0 || y < 0 || w < 1 || h < 1 || x + w > WIN || y + h > WIN)
                    PERR("line %d: rectangle outside the 24x24 window", cur.line);
                if (wt < -16 || wt > 16) PERR("line %d: weight outside [-16,16]", cur.line);
                sp->r[r].x = (int32_t)x; sp->r[r].y = (int32_t)y;
                sp->r[r].w = (int32_t)w; sp->r[r].h = (int32_t)h; sp->r[r].wt = (int32_t)wt;
            }
            if (!tok_float(&s, &sp->theta, 0) || !tok_float(&s, &sp->left, 0) || !tok_float(&s, &sp->right, 0) || !at_end(s))
                PERR("line %d: expected finite 'theta left right'", cur.line);
            c->n_stumps++;
        }
    }
    if (next_line(&cur, line, sizeof line)) PERR("line %d: trailing content", cur.line);
    if (c->packed) {
        /* encode every stump, then replace it by its decoded form: the cascade that is evaluated is
           the one the compressed words describe */
        c->words = (uint16_t*)malloc(sizeof(uint16_t) * (size_t)c->n_stumps * 9);
        if (!c->words) PERR("out of memory");
        for (int j = 0; j < c->n_stumps; ++j) {
            const int n = fdo_pack16(&c->stumps[j], c->words + c->n_words);
            if (n < 0) PERR("stump %d: not representable in packed16 (binary16 theta/left/right, fields)", j);
            fdo_unpack16(c->words + c->n_words, c->stumps[j].nrect, &c->stumps[j]);
            c->n_words += n;
        }
    }
    return c;
fail:
    fdo_cascade_free(c);
    return NULL;
}

/* ------------------------------------------------------------------------------------ */
/* c1: pyramid geometry ("n resized images", Fig. 2 fixed window P:L348-360)   */
/* ------------------------------------------------------------------------------------ */

int fdo_plan(int W, int H, int min_size, double scale, int step, int max_levels,
             double* f, int32_t* Wk, int32_t* Hk, int64_t* nwin) {
    if (W < WIN || H < WIN || min_size < WIN || !(scale > 1.0) || step < 1 || max_levels < 1) return -1;
    double fk = (double)min_size / 24.0;
    int n = 0;
    for (;;) {
        const int w = (int)floor((double)W / fk);
        const int h = (int)floor((double)H / fk);
        if (w < WIN || h < WIN) break;
        if (n == max_levels) return -1;
        f[n] = fk;
        Wk[n] = w;
        Hk[n] = h;
        nwin[n] = (int64_t)((w - WIN) / step + 1) * (int64_t)((h - WIN) / step + 1);
        ++n;
        fk = fk * scale;
    }
    return n;
}

/* ------------------------------------------------------------------------------------ */
/* c2: scaling -- each level sampled from the original frame, bilinear with  */
/* centre-aligned coordinates (x+1/2)f-1/2, 8-bit weights, clamp-to-edge; identity filter */
/* ------------------------------------------------------------------------------------ */

void fdo_resample(const uint8_t* frame, int W, int H, int pitch, double f, int Wk, int Hk, uint8_t* out) {
    const int64_t r = llround(f * 65536.0);
    for (int y = 0; y < Hk; ++y) {
        const int64_t sy = ((2 * (int64_t)y + 1) * r - 65536) >> 1;
        int y0 = (int)(sy >> 16);
        if (y0 > H - 1) y0 = H - 1;
        const int64_t ay = (sy >> 8) & 255;
        const int y1 = y0 + 1 < H ? y0 + 1 : H - 1;
        for (int x = 0; x < Wk; ++x) {
            const int64_t sx = ((2 * (int64_t)x + 1) * r - 65536) >> 1;
            int x0 = (int)(sx >> 16);
            if (x0 > W - 1) x0 = W - 1;
            const int64_t ax = (sx >> 8) & 255;
            const int x1 = x0 + 1 < W ? x0 + 1 : W - 1;
            const int64_t p00 = frame[(size_t)y0 * pitch + x0];
            const int64_t p01 = frame[(size_t)y0 * pitch + x1];
            const int64_t p10 = frame[(size_t)y1 * pitch + x0];
            const int64_t p11 = frame[(size_t)y1 * pitch + x1];
            const int64_t v = p00 * (256 - ax) * (256 - ay) + p01 * ax * (256 - ay) +
                              p10 * (256 - ax) * ay + p11 * ax * ay + 32768;
            out[(size_t)y * Wk + x] = (uint8_t)(v >> 16);
        }
    }
}

/* ------------------------------------------------------------------------------------ */
/* c3: integral and squared-integral images, padded exclusive    */
/* ------------------------------------------------------------------------------------ */

void fdo_integral(const uint8_t* img, int W, int H, int pitch, uint32_t* ii, uint64_t* sqii) {
    const int P = W + 1;
    for (int x = 0; x <= W; ++x) { ii[x] = 0; sqii[x] = 0; }
    for (int y = 0; y < H; ++y) {
        ii[(size_t)(y + 1) * P] = 0;
        sqii[(size_t)(y + 1) * P] = 0;
        for (int x = 0; x < W; ++x) {
            const uint32_t p = img[(size_t)y * pitch + x];
            ii[(size_t)(y + 1) * P + x + 1] = p + ii[(size_t)y * P + x + 1] + ii[(size_t)(y + 1) * P + x] - ii[(size_t)y * P + x];
            sqii[(size_t)(y + 1) * P + x + 1] = (uint64_t)p * p + sqii[(size_t)y * P + x + 1] +
                                                 sqii[(size_t)(y + 1) * P + x] - sqii[(size_t)y * P + x];
        }
    }
}

/* rect sum = A + D - B - C over the padded exclusive integral (Fig. 4 corner
 * pattern r[h0]+r[h1]-r[h2]-r[h3]) */
uint32_t fdo_rect_sum(const uint32_t* ii, int P, int x, int y, int w, int h) {
    const uint32_t A = ii[(size_t)y * P + x];
    const uint32_t B = ii[(size_t)y * P + x + w];
    const uint32_t C = ii[(size_t)(y + h) * P + x];
    const uint32_t D = ii[(size_t)(y + h) * P + x + w];
    return A + D - B - C;
}

static uint64_t rect_sum64(const uint64_t* ii, int P, int x, int y, int w, int h) {
    const uint64_t A = ii[(size_t)y * P + x];
    const uint64_t B = ii[(size_t)y * P + x + w];
    const uint64_t C = ii[(size_t)(y + h) * P + x];
    const uint64_t D = ii[(size_t)(y + h) * P + x + w];
    return A + D - B - C;
}

/* c5: variance normalisation over the full 24x24 window (Viola-Jones [7]):
 * v = N*Q - S^2 = N^2 sigma^2 (int64), nf = sqrtf((float)v) or 1 if v == 0 */
float fdo_window_nf(const uint32_t* ii, const uint64_t* sqii, int P, int wx, int wy) {
    const int64_t S = (int64_t)fdo_rect_sum(ii, P, wx, wy, WIN, WIN);
    const int64_t Q = (int64_t)rect_sum64(sqii, P, wx, wy, WIN, WIN);
    const int64_t v = (int64_t)WIN_AREA * Q - S * S;
    return v > 0 ? sqrtf((float)v) : 1.0f;
}

/* c6: Haar feature response f = sum_r wt_r * R_r (9 accesses per rectangle) */
int32_t fdo_feature(const uint32_t* ii, int P, int wx, int wy, const fdo_rect* r, int nrect) {
    int64_t f = 0;
    for (int i = 0; i < nrect; ++i)
        f += (int64_t)r[i].wt * (int64_t)fdo_rect_sum(ii, P, wx + r[i].x, wy + r[i].y, r[i].w, r[i].h);
    return (int32_t)f;
}

void fdo_feature_values(const uint32_t* ii, int P, const int32_t* wins, int64_t nw,
                        const fdo_rect* r, int nrect, int32_t* out) {
    for (int64_t i = 0; i < nw; ++i) out[i] = fdo_feature(ii, P, wins[2 * i], wins[2 * i + 1], r, nrect);
}

void fdo_window_nf_values(const uint32_t* ii, const uint64_t* sqii, int P,
                          const int32_t* wins, int64_t nw, float* out) {
    for (int64_t i = 0; i < nw; ++i) out[i] = fdo_window_nf(ii, sqii, P, wins[2 * i], wins[2 * i + 1]);
}

/* c7 stump (GentleBoost regression stump [6]) and c8 stages with early
 * rejection: sum = sum + leaf in stump order (fp32), pass iff sum >= T.
 * Soft cascade (f4; the paper's future work, ref [32] Bourdev & Brandt; reading
 * R8b): the sum is NOT restarted at a stage boundary -- it runs over every stump evaluated so
 * far and T_s is the rejection threshold of the running sum after stage s (one-stump stages
 * give the per-stump rejection trace of [32]). */
int fdo_eval_window(const fdo_cascade* c, const uint32_t* ii, const uint64_t* sqii, int P,
                    int wx, int wy, float* score, int* near) {
    const float nf = fdo_window_nf(ii, sqii, P, wx, wy);
    int nr = 0;
    float sum = 0.0f;
    for (int s = 0; s < c->n_stages; ++s) {
        const fdo_stage* st = &c->stages[s];
        if (!c->soft) sum = 0.0f;
        for (int j = 0; j < st->n; ++j) {
            const fdo_stump* sp = &c->stumps[st->first + j];
            const int32_t f = fdo_feature(ii, P, wx, wy, sp->r, sp->nrect);
            const float t = sp->theta * nf;
            const float ff = (float)f;
            const float leaf = (ff < t) ? sp->left : sp->right;
            if (fabs((double)ff - (double)t) <= 1e-4 * fmax(1.0, fabs((double)t))) nr |= 2;
            sum = sum + leaf;
        }
        if (isfinite(st->T) && fabs((double)sum - (double)st->T) <= 1e-4) nr |= 1;
        if (!(sum >= st->T)) {
            *score = sum;
            *near = nr;
            return s;
        }
    }
    *score = sum;
    *near = nr;
    return c->n_stages;
}

void fdo_eval_level(const fdo_cascade* c, const uint32_t* ii, const uint64_t* sqii, int Wk, int Hk,
                    int step, uint8_t* depth, float* score, uint8_t* near) {
    const int P = Wk + 1;
    const int nx = (Wk - WIN) / step + 1, ny = (Hk - WIN) / step + 1;
    for (int j = 0; j < ny; ++j)
        for (int i = 0; i < nx; ++i) {
            float sc;
            int nr;
            const int d = fdo_eval_window(c, ii, sqii, P, i * step, j * step, &sc, &nr);
            const size_t o = (size_t)j * nx + i;
            depth[o] = (uint8_t)(d > 255 ? 255 : d);
            score[o] = sc;
            if (near) near[o] = (uint8_t)nr;
        }
}

/* ------------------------------------------------------------------------------------ */
/* f2: filtering stage (P:L362-367 names it, gives no taps; reading R3b): binomial 3x3,     */
/* out(x,y) = (sum_{i,j in -1..1} w_i w_j in(clamp(x+i), clamp(y+j)) + 8) >> 4,              */
/* w_-1 = w_1 = 1, w_0 = 2, written out directly (no separable pass, no reordering).         */
/* ------------------------------------------------------------------------------------ */

void fdo_filter_binomial(uint8_t* img, int W, int H) {
    static const int w[3] = {1, 2, 1};
    uint8_t* src = (uint8_t*)malloc((size_t)W * H);
    if (!src) return;
    memcpy(src, img, (size_t)W * H);
    for (int y = 0; y < H; ++y)
        for (int x = 0; x < W; ++x) {
            int sum = 0;
            for (int j = -1; j <= 1; ++j)
                for (int i = -1; i <= 1; ++i) {
                    int xx = x + i, yy = y + j;
                    if (xx < 0) xx = 0;
                    if (xx > W - 1) xx = W - 1;
                    if (yy < 0) yy = 0;
                    if (yy > H - 1) yy = H - 1;
                    sum += w[i + 1] * w[j + 1] * src[(size_t)yy * W + xx];
                }
            img[(size_t)y * W + x] = (uint8_t)((sum + 8) >> 4);
        }
    free(src);
}

/* ------------------------------------------------------------------------------------ */
/* Whole path over frames: jobs = (frame, level), run on host threads, merged in order.  */
/* ------------------------------------------------------------------------------------ */

typedef struct {
    const fdo_cascade* c;
    const uint8_t* frames;
    int n, W, H, pitch, step, nl;
    double f[FDO_MAX_LEVELS];
    int32_t Wk[FDO_MAX_LEVELS], Hk[FDO_MAX_LEVELS];
    int64_t nwin[FDO_MAX_LEVELS], lvl_off[FDO_MAX_LEVELS + 1];
    /* depth mode */
    uint8_t* depth; float* score; uint8_t* near;
    /* detect mode: per job results */
    fdo_detection** job_det; int64_t* job_cnt; int64_t* job_near;
    int next; pthread_mutex_t mu; int err;
} run_t;

static void run_job(run_t* R, int job) {
    const int fr = job / R->nl, k = job % R->nl;
    const int Wk = R->Wk[k], Hk = R->Hk[k], P = Wk + 1;
    const uint8_t* frame = R->frames + (size_t)fr * R->pitch * R->H;
    uint8_t* lvl = (uint8_t*)malloc((size_t)Wk * Hk);
    uint32_t* ii = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)P * (Hk + 1));
    uint64_t* sq = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)P * (Hk + 1));
    const int nx = (Wk - WIN) / R->step + 1, ny = (Hk - WIN) / R->step + 1;
    uint8_t* dep = NULL; float* sco = NULL; uint8_t* nr = NULL;
    int own = 0;
    if (R->depth) {
        const size_t o = (size_t)fr * R->lvl_off[R->nl] + R->lvl_off[k];
        dep = R->depth + o; sco = R->score + o; nr = R->near ? R->near + o : NULL;
    } else {
        dep = (uint8_t*)malloc((size_t)nx * ny);
        sco = (float*)malloc(sizeof(float) * (size_t)nx * ny);
        nr = (uint8_t*)malloc((size_t)nx * ny);
        own = 1;
    }
    if (!lvl || !ii || !sq || !dep || !sco || (own && !nr)) {
        R->err = 1;
        goto done;
    }
    fdo_resample(frame, R->W, R->H, R->pitch, R->f[k], Wk, Hk, lvl);
    if (R->c->filter) fdo_filter_binomial(lvl, Wk, Hk);
    fdo_integral(lvl, Wk, Hk, Wk, ii, sq);
    fdo_eval_level(R->c, ii, sq, Wk, Hk, R->step, dep, sco, nr);
    if (own) {
        int64_t cnt = 0, nnear = 0;
        for (int64_t i = 0; i < (int64_t)nx * ny; ++i) {
            if (dep[i] == R->c->n_stages) ++cnt;
            if (nr[i]) ++nnear;
        }
        fdo_detection* d = (fdo_detection*)malloc(sizeof(fdo_detection) * (size_t)(cnt ? cnt : 1));
        if (!d) { R->err = 1; goto done; }
        int64_t q = 0;
        const double fk = R->f[k];
        for (int j = 0; j < ny; ++j)
            for (int i = 0; i < nx; ++i) {
                const size_t o = (size_t)j * nx + i;
                if (dep[o] != R->c->n_stages) continue;
                /* c9: back-projection, size = factor x 24, round half up */
                const int wx = i * R->step, wy = j * R->step;
                d[q].frame = fr; d[q].level = k; d[q].wx = wx; d[q].wy = wy;
                d[q].x = (int32_t)floor(wx * fk + 0.5);
                d[q].y = (int32_t)floor(wy * fk + 0.5);
                d[q].w = (int32_t)floor(24.0 * fk + 0.5);
                d[q].h = d[q].w;
                d[q].score = sco[o];
                d[q].aux = R->c->n_stages;
                ++q;
            }
        R->job_det[job] = d;
        R->job_cnt[job] = cnt;
        R->job_near[job] = nnear;
    }
done:
    free(lvl); free(ii); free(sq);
    if (own) { free(dep); free(sco); free(nr); }
}

static void* run_worker(void* arg) {
    run_t* R = (run_t*)arg;
    for (;;) {
        pthread_mutex_lock(&R->mu);
        const int j = R->next++;
        pthread_mutex_unlock(&R->mu);
        if (j >= R->n * R->nl) break;
        run_job(R, j);
    }
    return NULL;
}

static int run_all(run_t* R, int nthreads) {
    pthread_mutex_init(&R->mu, NULL);
    R->next = 0;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 512) nthreads = 512;
    pthread_t th[512];
    int started = 0;
    for (int t = 1; t < nthreads; ++t)
        if (pthread_create(&th[started], NULL, run_worker, R) == 0) ++started;
    run_worker(R);
    for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
    pthread_mutex_destroy(&R->mu);
    return R->err ? -1 : 0;
}

static int run_init(run_t* R, const fdo_cascade* c, const uint8_t* frames, int n, int W, int H, int pitch,
                    int min_size, double scale, int step) {
    memset(R, 0, sizeof *R);
    if (!c || !frames || n < 1 || pitch < W) return -1;
    R->c = c; R->frames = frames; R->n = n; R->W = W; R->H = H; R->pitch = pitch; R->step = step;
    R->nl = fdo_plan(W, H, min_size, scale, step, FDO_MAX_LEVELS, R->f, R->Wk, R->Hk, R->nwin);
    if (R->nl < 0) return -1;
    R->lvl_off[0] = 0;
    for (int k = 0; k < R->nl; ++k) R->lvl_off[k + 1] = R->lvl_off[k] + R->nwin[k];
    return 0;
}

int fdo_detect_depth(const fdo_cascade* c, const uint8_t* frames, int n, int W, int H, int pitch,
                     int min_size, double scale, int step, int nthreads,
                     uint8_t* depth, float* score, uint8_t* near) {
    run_t* R = (run_t*)malloc(sizeof(run_t));
    if (!R) return -1;
    if (run_init(R, c, frames, n, W, H, pitch, min_size, scale, step) != 0 || !depth || !score) { free(R); return -1; }
    R->depth = depth; R->score = score; R->near = near;
    const int rc = R->nl > 0 ? run_all(R, nthreads) : 0;
    free(R);
    return rc;
}

int64_t fdo_detect(const fdo_cascade* c, const uint8_t* frames, int n, int W, int H, int pitch,
                   int min_size, double scale, int step, int nthreads,
                   fdo_detection* out, int64_t cap, int64_t* n_near) {
    run_t* R = (run_t*)malloc(sizeof(run_t));
    if (!R) return -1;
    if (run_init(R, c, frames, n, W, H, pitch, min_size, scale, step) != 0) { free(R); return -1; }
    const int nj = n * R->nl;
    if (nj == 0) { if (n_near) *n_near = 0; free(R); return 0; }
    R->job_det = (fdo_detection**)calloc((size_t)nj, sizeof(fdo_detection*));
    R->job_cnt = (int64_t*)calloc((size_t)nj, sizeof(int64_t));
    R->job_near = (int64_t*)calloc((size_t)nj, sizeof(int64_t));
    int64_t total = -1;
    if (R->job_det && R->job_cnt && R->job_near && run_all(R, nthreads) == 0) {
        /* jobs are (frame, level)-ordered and each job emits (wy, wx) order: already sorted */
        total = 0;
        int64_t nn = 0;
        for (int j = 0; j < nj; ++j) {
            for (int64_t i = 0; i < R->job_cnt[j]; ++i) {
                if (total < cap && out) out[total] = R->job_det[j][i];
                ++total;
            }
            nn += R->job_near[j];
        }
        if (n_near) *n_near = nn;
    }
    if (R->job_det) for (int j = 0; j < nj; ++j) free(R->job_det[j]);
    free(R->job_det); free(R->job_cnt); free(R->job_near);
    free(R);
    return total;
}

/* ------------------------------------------------------------------------------------ */
/* c10: grouping with the eyes metric, eq. 6 and the merge rule            */
/* "overlap whenever S_eyes(d_i,d_j) < 0.5 ... progressively averaging those with the     */
/* highest overlapping".  Eye template (0.3,0.4)/(0.7,0.4) of the window.  */
/* ------------------------------------------------------------------------------------ */

typedef struct { double lex, ley, rex, rey, d; } eyes_t;

static eyes_t eyes_of(double mx, double my, double mw, double mh) {
    eyes_t e;
    e.lex = mx + 0.3 * mw;
    e.ley = my + 0.4 * mh;
    e.rex = mx + 0.7 * mw;
    e.rey = my + 0.4 * mh;
    e.d = sqrt((e.rex - e.lex) * (e.rex - e.lex) + (e.rey - e.ley) * (e.rey - e.ley));
    return e;
}

static double s_eyes_e(eyes_t a, eyes_t b) {
    const double dle = sqrt((a.lex - b.lex) * (a.lex - b.lex) + (a.ley - b.ley) * (a.ley - b.ley));
    const double dre = sqrt((a.rex - b.rex) * (a.rex - b.rex) + (a.rey - b.rey) * (a.rey - b.rey));
    const double m = a.d < b.d ? a.d : b.d;
    return (dle + dre) / m;
}

double fdo_s_eyes(double ax, double ay, double aw, double ah, double bx, double by, double bw, double bh) {
    return s_eyes_e(eyes_of(ax, ay, aw, ah), eyes_of(bx, by, bw, bh));
}

typedef struct { int64_t sx, sy, sw, sh, n; float smax; int first; int active; } cluster_t;

static eyes_t cluster_eyes(const cluster_t* c) {
    const double n = (double)c->n;
    return eyes_of((double)c->sx / n, (double)c->sy / n, (double)c->sw / n, (double)c->sh / n);
}

int64_t fdo_group(const fdo_detection* in, int64_t n, double eyes_thresh, int min_neighbors,
                  fdo_detection* out, int64_t cap) {
    int64_t total = 0, a = 0;
    while (a < n) {
        int64_t b = a;
        while (b < n && in[b].frame == in[a].frame) ++b;
        const int64_t m = b - a;
        cluster_t* cl = (cluster_t*)malloc(sizeof(cluster_t) * (size_t)m);
        if (!cl) return -1;
        for (int64_t i = 0; i < m; ++i) {
            const fdo_detection* d = &in[a + i];
            cl[i].sx = d->x; cl[i].sy = d->y; cl[i].sw = d->w; cl[i].sh = d->h;
            cl[i].n = 1; cl[i].smax = d->score; cl[i].first = (int)i; cl[i].active = 1;
        }
        for (;;) {
            double best = INFINITY;
            int64_t bi = -1, bj = -1;
            for (int64_t i = 0; i < m; ++i) {
                if (!cl[i].active) continue;
                const eyes_t ei = cluster_eyes(&cl[i]);
                for (int64_t j = i + 1; j < m; ++j) {
                    if (!cl[j].active) continue;
                    const double s = s_eyes_e(ei, cluster_eyes(&cl[j]));
                    if (s < best) { best = s; bi = i; bj = j; }
                }
            }
            if (bi < 0 || !(best < eyes_thresh)) break;
            cl[bi].sx += cl[bj].sx; cl[bi].sy += cl[bj].sy; cl[bi].sw += cl[bj].sw; cl[bi].sh += cl[bj].sh;
            cl[bi].n += cl[bj].n;
            if (cl[bj].smax > cl[bi].smax) cl[bi].smax = cl[bj].smax;
            cl[bj].active = 0;
        }
        for (int64_t i = 0; i < m; ++i) {
            if (!cl[i].active || cl[i].n < min_neighbors) continue;
            if (total < cap && out) {
                const fdo_detection* d0 = &in[a + cl[i].first];
                fdo_detection* o = &out[total];
                const double nn = (double)cl[i].n;
                o->frame = d0->frame; o->level = d0->level; o->wx = d0->wx; o->wy = d0->wy;
                o->x = (int32_t)floor((double)cl[i].sx / nn + 0.5);
                o->y = (int32_t)floor((double)cl[i].sy / nn + 0.5);
                o->w = (int32_t)floor((double)cl[i].sw / nn + 0.5);
                o->h = (int32_t)floor((double)cl[i].sh / nn + 0.5);
                o->score = cl[i].smax;
                o->aux = (int32_t)cl[i].n;
            }
            ++total;
        }
        free(cl);
        a = b;
    }
    return total;
}
