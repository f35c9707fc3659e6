/*
 * fdgen.c -- seeded synthetic workload generator (frames, face template, planting).
 *
 * This module is INPUT GENERATION ONLY.  It holds none of the face-detection
 * method's arithmetic (no pyramid resampling, no integral images, no feature or
 * cascade evaluation).  Both the CPU oracle (oracle/) and the CUDA path
 * (paper_conf_icpp_orofsmh12_b200/) consume its frames; neither is linked in.
 *
 * Recipe (after SURVEY.md 8(d)):
 *   - PRNG: splitmix64, counter based.  frame seed = mix(0xFD00 + cfg, frame index),
 *     so a frame's bytes depend only on (cfg, global frame index), never on the
 *     number of GPUs or the batch it is generated in.
 *   - background: mean 128 + 3 octaves of value noise (cells 64/16/4 px,
 *     amplitudes 60/30/15 grey levels, bilinear in Q8), + uniform [-8,8] per-pixel
 *     noise, x per-frame contrast jitter in [0.8,1.2] (Q8), clamped to [0,255].
 *     Integer arithmetic only, so every machine produces identical bytes.
 *   - template: 24x24 binary "face-like" pattern, values 20 / 235
 *     (paper: 24x24 frontal faces, section IV).
 *   - planted faces: rendered (nearest neighbour) at size S = floor(24 f + 1/2) at
 *     (floor(wx f + 1/2), floor(wy f + 1/2)) for a caller-supplied pyramid scale f
 *     and window origin (wx, wy) on that level's grid; non-overlapping.
 *     The caller passes the level table (f, W_k, H_k); this module does not derive it.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline uint64_t sm64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
static inline uint64_t h2(uint64_t a, uint64_t b) { return sm64(a ^ sm64(b)); }
static inline uint64_t h3(uint64_t a, uint64_t b, uint64_t c) { return h2(h2(a, b), c); }
static inline uint64_t h4(uint64_t a, uint64_t b, uint64_t c, uint64_t d) { return h2(h3(a, b, c), d); }

uint64_t fdgen_splitmix64(uint64_t x) { return sm64(x); }

uint64_t fdgen_frame_seed(uint32_t cfg, uint64_t frame_index) {
    return h2(0xFD00ULL + (uint64_t)cfg, frame_index);
}

/* 24x24 template: 1 = bright (235), 0 = dark (20). Rows top->bottom. */
static const char* TEMPLATE_ROWS[24] = {
    "000000000000000000000000",  /*  0 hair            */
    "000000000000000000000000",  /*  1 hair            */
    "001111111111111111111100",  /*  2 forehead        */
    "011111111111111111111110",  /*  3                 */
    "011111111111111111111110",  /*  4                 */
    "011111111111111111111110",  /*  5                 */
    "011111111111111111111110",  /*  6                 */
    "010000000011110000000010",  /*  7 eye band        */
    "010000000011110000000010",  /*  8                 */
    "010000000011110000000010",  /*  9                 */
    "011111111111111111111110",  /* 10                 */
    "011111111111111111111110",  /* 11 cheeks / nose   */
    "011111111100001111111110",  /* 12                 */
    "011111111100001111111110",  /* 13                 */
    "011111111111111111111110",  /* 14                 */
    "011111111111111111111110",  /* 15                 */
    "011111000000000000111110",  /* 16 mouth           */
    "011111000000000000111110",  /* 17                 */
    "011111000000000000111110",  /* 18                 */
    "011111111111111111111110",  /* 19                 */
    "001111111111111111111100",  /* 20 chin            */
    "000111111111111111111000",  /* 21                 */
    "000011111111111111110000",  /* 22                 */
    "000000000000000000000000",  /* 23                 */
};

void fdgen_template(uint8_t out[576]) {
    for (int y = 0; y < 24; ++y)
        for (int x = 0; x < 24; ++x)
            out[y * 24 + x] = TEMPLATE_ROWS[y][x] == '1' ? 235 : 20;
}

/* value-noise lattice for one octave: (gw x gh) values in [-256, 256] */
static void lattice(uint64_t fs, int oct, int gw, int gh, int32_t* L) {
    for (int j = 0; j < gh; ++j)
        for (int i = 0; i < gw; ++i)
            L[j * gw + i] = (int32_t)((h4(fs, 100 + oct, (uint64_t)i, (uint64_t)j) >> 40) % 513) - 256;
}

/* Background only. Returns 0 on success, -1 on allocation failure. */
int fdgen_background(uint32_t cfg, uint64_t frame_index, int W, int H, int pitch, uint8_t* out) {
    static const int CELL_LOG2[3] = {6, 4, 2};
    static const int64_t AMP[3] = {60, 30, 15};
    const uint64_t fs = fdgen_frame_seed(cfg, frame_index);
    int32_t* L[3];
    int gw[3], gh[3];
    for (int o = 0; o < 3; ++o) {
        gw[o] = (W >> CELL_LOG2[o]) + 2;
        gh[o] = (H >> CELL_LOG2[o]) + 2;
        L[o] = (int32_t*)malloc(sizeof(int32_t) * (size_t)gw[o] * (size_t)gh[o]);
        if (!L[o]) { for (int q = 0; q < o; ++q) free(L[q]); return -1; }
        lattice(fs, o, gw[o], gh[o], L[o]);
    }
    const int64_t cj = 205 + (int64_t)(h2(fs, 4) % 103);   /* contrast jitter, Q8: 0.80..1.20 */
    for (int y = 0; y < H; ++y) {
        for (int x = 0; x < W; ++x) {
            int64_t acc = 0;
            for (int o = 0; o < 3; ++o) {
                const int cl = CELL_LOG2[o];
                const int i = x >> cl, j = y >> cl;
                const int64_t wx = (int64_t)(x & ((1 << cl) - 1)) << (8 - cl);
                const int64_t wy = (int64_t)(y & ((1 << cl) - 1)) << (8 - cl);
                const int32_t* Lo = L[o];
                const int64_t l00 = Lo[j * gw[o] + i], l10 = Lo[j * gw[o] + i + 1];
                const int64_t l01 = Lo[(j + 1) * gw[o] + i], l11 = Lo[(j + 1) * gw[o] + i + 1];
                const int64_t v = l00 * (256 - wx) * (256 - wy) + l10 * wx * (256 - wy) +
                                  l01 * (256 - wx) * wy + l11 * wx * wy;      /* |v| <= 2^24 */
                acc += AMP[o] * v;
            }
            const int64_t noise = (int64_t)((h4(fs, 3, (uint64_t)x, (uint64_t)y) >> 40) % 17) - 8;
            const int64_t d = ((acc + (1LL << 23)) >> 24) + noise;
            int64_t p = 128 + ((d * cj) >> 8);
            if (p < 0) p = 0;
            if (p > 255) p = 255;
            out[(size_t)y * (size_t)pitch + (size_t)x] = (uint8_t)p;
        }
    }
    for (int o = 0; o < 3; ++o) free(L[o]);
    return 0;
}

/* Render the template at size S with top-left (X, Y) (nearest neighbour). */
void fdgen_render_face(uint8_t* out, int W, int H, int pitch, int X, int Y, int S) {
    uint8_t T[576];
    fdgen_template(T);
    for (int v = 0; v < S; ++v) {
        const int yy = Y + v;
        if (yy < 0 || yy >= H) continue;
        const int ty = (int)(((int64_t)v * 24) / S);
        for (int u = 0; u < S; ++u) {
            const int xx = X + u;
            if (xx < 0 || xx >= W) continue;
            const int tx = (int)(((int64_t)u * 24) / S);
            out[(size_t)yy * (size_t)pitch + (size_t)xx] = T[ty * 24 + tx];
        }
    }
}

/* Poisson draw from a uniform in [0,1): inversion with an IEEE-only recurrence. */
static int poisson4(uint64_t hbits, double mean) {
    /* e^-mean computed by repeated multiplication of e^-1/4 so only + * / are used */
    const double E_M025 = 0.77880078307140486824;          /* e^-0.25 */
    double p = 1.0;
    int q = (int)(mean * 4.0 + 0.5);
    for (int i = 0; i < q; ++i) p *= E_M025;
    const double u = (double)(hbits >> 11) * (1.0 / 9007199254740992.0);
    double cdf = p;
    int k = 0;
    while (u > cdf && k < 64) { ++k; p *= mean / (double)k; cdf += p; }
    return k;
}

/*
 * Full frame: background + planted faces.
 *   face_mode 0: none; 1: exactly `face_param` faces; 2: Poisson(face_param) faces.
 *   levels (f, Wk, Hk)[n_levels] come from the caller's pyramid plan; faces are only
 *   placed on levels k < max_face_level with a window grid point (wx, wy).
 *   faces_out[i*6 + {0..5}] = level, wx, wy, X, Y, S.  Returns number of faces, or -1.
 */
int fdgen_frame(uint32_t cfg, uint64_t frame_index, int W, int H, int pitch, uint8_t* out,
                int n_levels, const double* f, const int* Wk, const int* Hk, int max_face_level,
                int face_mode, double face_param, int32_t* faces_out, int max_faces) {
    if (fdgen_background(cfg, frame_index, W, H, pitch, out) != 0) return -1;
    if (face_mode == 0 || n_levels <= 0) return 0;
    const uint64_t fs = fdgen_frame_seed(cfg, frame_index);
    int want = face_mode == 1 ? (int)face_param : poisson4(h2(fs, 5), face_param);
    if (want > max_faces) want = max_faces;
    int nl = n_levels < max_face_level ? n_levels : max_face_level;
    if (nl <= 0) return 0;
    int nf = 0;
    for (int attempt = 0; attempt < 64 * (want + 1) && nf < want; ++attempt) {
        const uint64_t r = h3(fs, 6, (uint64_t)attempt);
        const int k = (int)(r % (uint64_t)nl);
        const int rx = Wk[k] - 24 + 1, ry = Hk[k] - 24 + 1;
        if (rx <= 0 || ry <= 0) continue;
        const int wx = (int)(h3(fs, 7, (uint64_t)attempt) % (uint64_t)rx);
        const int wy = (int)(h3(fs, 8, (uint64_t)attempt) % (uint64_t)ry);
        const double fk = f[k];
        const int X = (int)(wx * fk + 0.5), Y = (int)(wy * fk + 0.5), S = (int)(24.0 * fk + 0.5);
        if (X + S > W || Y + S > H) continue;
        int clash = 0;
        for (int q = 0; q < nf; ++q) {   /* keep a 1/4-size gap between planted faces */
            const int32_t* o = faces_out + 6 * q;
            const int g = (S > o[5] ? S : o[5]) / 4;
            if (X < o[3] + o[5] + g && o[3] < X + S + g && Y < o[4] + o[5] + g && o[4] < Y + S + g) { clash = 1; break; }
        }
        if (clash) continue;
        int32_t* o = faces_out + 6 * nf;
        o[0] = k; o[1] = wx; o[2] = wy; o[3] = X; o[4] = Y; o[5] = S;
        ++nf;
    }
    for (int q = 0; q < nf; ++q) {
        const int32_t* o = faces_out + 6 * q;
        fdgen_render_face(out, W, H, pitch, o[3], o[4], o[5]);
    }
    return nf;
}

/* ---- batch generation over threads (frames are independent) ---- */
#include <pthread.h>
typedef struct {
    uint32_t cfg; uint64_t first; int n, W, H, pitch; uint8_t* out;
    int n_levels; const double* f; const int* Wk; const int* Hk; int max_face_level;
    int face_mode; double face_param; int32_t* faces; int32_t* nfaces; int max_faces;
    int next; pthread_mutex_t mu; int err;
} batch_t;

static void* batch_worker(void* arg) {
    batch_t* b = (batch_t*)arg;
    for (;;) {
        pthread_mutex_lock(&b->mu);
        const int i = b->next++;
        pthread_mutex_unlock(&b->mu);
        if (i >= b->n) break;
        const int r = fdgen_frame(b->cfg, b->first + (uint64_t)i, b->W, b->H, b->pitch,
                                  b->out + (size_t)i * (size_t)b->pitch * (size_t)b->H,
                                  b->n_levels, b->f, b->Wk, b->Hk, b->max_face_level,
                                  b->face_mode, b->face_param,
                                  b->faces ? b->faces + (size_t)i * 6 * (size_t)b->max_faces : NULL,
                                  b->max_faces);
        if (r < 0) b->err = 1;
        if (b->nfaces) b->nfaces[i] = r < 0 ? 0 : r;
    }
    return NULL;
}

/* n frames with global indices first..first+n-1 into out[n][H][pitch]; faces[n][max_faces][6]. */
int fdgen_frames(uint32_t cfg, uint64_t first, int n, int W, int H, int pitch, uint8_t* out,
                 int n_levels, const double* f, const int* Wk, const int* Hk, int max_face_level,
                 int face_mode, double face_param, int32_t* faces, int32_t* nfaces, int max_faces,
                 int nthreads) {
    batch_t b;
    int32_t dummy[6 * 64];
    b.cfg = cfg; b.first = first; b.n = n; b.W = W; b.H = H; b.pitch = pitch; b.out = out;
    b.n_levels = n_levels; b.f = f; b.Wk = Wk; b.Hk = Hk; b.max_face_level = max_face_level;
    b.face_mode = faces ? face_mode : 0; b.face_param = face_param; b.faces = faces; b.nfaces = nfaces;
    b.max_faces = faces ? max_faces : 0; b.next = 0; b.err = 0;
    (void)dummy;
    pthread_mutex_init(&b.mu, NULL);
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    pthread_t th[256];
    int started = 0;
    for (int t = 1; t < nthreads; ++t)
        if (pthread_create(&th[started], NULL, batch_worker, &b) == 0) ++started;
    batch_worker(&b);
    for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
    pthread_mutex_destroy(&b.mu);
    return b.err ? -1 : 0;
}
