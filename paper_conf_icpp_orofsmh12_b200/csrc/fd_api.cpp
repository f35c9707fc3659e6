// fd_api.cpp -- the C ABI (include/fd.h): validation, pyramid plan, cascade parsing and
// packing, per-(device, stream) workspaces, and the launch sequence of the hot path, per frame
// group on two pipeline slots:
//   default (f1):  k_level (level images, u8)  ->  k_f1 (persistent, all scales: tile-local
//                  integral + every stage)  ->  k_tail
//   FD_F1=0 / soft cascades:  K1 (k_marg -> k_carry/k_corner -> k_tile: global ii + sqii)
//                  ->  k_stage1 + k_deep1 (+ k_tail), or k_soft
//   then count read-back -> K3 (radix sort + back-projection).
// Host code only; every arithmetic step of the method runs in the kernels.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cerrno>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "fd_internal.h"
#include "fd_jit.h"

using namespace fdk;

namespace {

thread_local std::string g_err;

fd_status fail(fd_status s, const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return s;
}

#define CK(expr)                                                                                  \
    do {                                                                                          \
        cudaError_t e_ = (expr);                                                                  \
        if (e_ != cudaSuccess) return fail(FD_ECUDA, "%s: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

// ------------------------------------------------------------------ pyramid plan (reading R1)
fd_status make_plan(int W, int H, int min_size, double s, int step, fd_plan* out) {
    if (W < WIN || H < WIN) return fail(FD_EINVAL, "frame %dx%d smaller than the 24x24 window", W, H);
    if (min_size < WIN) return fail(FD_EINVAL, "min_size %d < 24", min_size);
    if (!(s > 1.0) || !std::isfinite(s)) return fail(FD_EINVAL, "scale_factor must be > 1");
    if (step < 1) return fail(FD_EINVAL, "step must be >= 1");
    if (W > 65535 || H > 65535) return fail(FD_EINVAL, "frame larger than 65535");
    std::memset(out, 0, sizeof *out);
    double f = (double)min_size / 24.0;
    int n = 0;
    for (;;) {
        const int w = (int)std::floor((double)W / f);
        const int h = (int)std::floor((double)H / f);
        if (w < WIN || h < WIN) break;
        if (n == FD_MAX_LEVELS) return fail(FD_EINVAL, "more than %d pyramid levels", FD_MAX_LEVELS);
        out->f[n] = f;
        out->w[n] = w;
        out->h[n] = h;
        out->windows[n] = (int64_t)((w - WIN) / step + 1) * (int64_t)((h - WIN) / step + 1);
        out->total_windows += out->windows[n];
        ++n;
        f = f * s;
    }
    out->n_levels = n;
    return FD_OK;
}

// device plan for a frame group of G frames
void make_plan_dev(const fd_plan& pl, int W, int H, int pitch, int step, int G, PlanDev* p) {
    std::memset(p, 0, sizeof *p);
    p->n_levels = pl.n_levels;
    p->W = W;
    p->H = H;
    p->pitch = pitch;
    p->step = step;
    p->G = G;
    const int tx = k2_tx(step), ty = k2_ty(step);
    long long ws = 0, col = 0, win = 0, row = 0, cor = 0, lvl = 0, u8 = 0;
    int bands = 0, tiles = 0, maxW = 0, k1t = 0;
    for (int k = 0; k < pl.n_levels; ++k) {
        LevelDev& L = p->lv[k];
        L.W = pl.w[k];
        L.H = pl.h[k];
        L.P = (L.W + 1 + 3) & ~3;
        L.PB = (L.W + 1 + 15) & ~15;
        L.u8_off = u8;
        u8 += (long long)G * L.H * L.PB;
        L.nx = (L.W - WIN) / step + 1;
        L.ny = (L.H - WIN) / step + 1;
        L.band0 = bands;
        L.nbands = (L.H + BAND - 1) / BAND;
        L.tile0 = tiles;
        L.tiles_x = (L.nx + tx - 1) / tx;
        L.r16 = (int)std::llround(pl.f[k] * 65536.0);
        L.nchunks = (L.P + CHUNK - 1) / CHUNK;
        L.k1t0 = k1t;
        L.ws_off = ws;
        L.col_off = col;
        L.row_off = row;
        L.cor_off = cor;
        L.lvl_off = lvl;
        L.win0 = win;
        lvl += (long long)L.H * L.PB;
        bands += L.nbands;
        k1t += L.nbands * L.nchunks;
        tiles += L.tiles_x * ((L.ny + ty - 1) / ty);
        ws += (long long)G * 2 * (L.H + 1) * L.P;
        col += (long long)L.nbands * 2 * L.W;
        row += (long long)L.nbands * L.nchunks * 2 * BAND;
        cor += (long long)L.nbands * L.nchunks * 2;
        win += pl.windows[k];
        maxW = L.W > maxW ? L.W : maxW;
    }
    p->bands_per_frame = bands;
    p->tiles_per_frame = tiles;
    p->k1tiles_per_frame = k1t;
    p->maxW = maxW;
    p->win_per_frame = win;
    p->col_frame = col;
    p->row_frame = row;
    p->cor_frame = cor;
    p->lvl_frame = lvl;
    p->ws_elems = ws;
    p->u8_bytes = u8;
}

// ------------------------------------------------------------------ cascade (.fdc) parser
struct HStump {
    int nrect;
    int r[3][5];
    float theta, left, right;
};
struct HStage {
    int first, n;
    float T;
};

struct Line {
    std::vector<std::string> tok;
    int no;
};

bool parse_int(const std::string& t, long* v) {
    char* e = nullptr;
    errno = 0;
    *v = std::strtol(t.c_str(), &e, 10);
    return e && *e == 0 && errno == 0 && !t.empty();
}
bool parse_float(const std::string& t, float* v, bool allow_inf) {
    char* e = nullptr;
    *v = std::strtof(t.c_str(), &e);
    if (!e || *e != 0 || t.empty()) return false;
    if (std::isnan(*v)) return false;
    if (!allow_inf && std::isinf(*v)) return false;
    return true;
}

}  // namespace

struct fd_cascade_s {
    int device = 0;
    int filter = 0;                         // filtering stage after scaling: 0 none, 1 binomial 3x3
    int soft = 0;                           // 1: soft cascade (f4, reading R8b), stage sums carried over
    int compressed = 0;                     // 1: 'compress packed16' (f3, reading R13)
    std::vector<uint32_t> pk16;             // f3: FD_PK_WORDS u32 per stump (rects: two 16-bit words each)
    std::vector<HStump> stumps;
    std::vector<HStage> stages;
    std::mutex mu;
    struct Packed {
        uint4* d_rec = nullptr;             // device records (REC_WORDS u32 per stump)
        StageDev* d_st = nullptr;
        uint32_t* d_trec = nullptr;         // SoA tail records (k_tail): [TAIL_REC_WORDS][n_stumps]
        std::vector<uint32_t> h_rec;        // host copy (first PREC_MAX go to the parameter bank)
        std::vector<StageDev> h_st;         // host copy (first PSTAGE_MAX go to the parameter bank)
    };
    std::map<int, Packed> packed;           // tile width -> packed records
    fdk::JitK2* jit = nullptr;              // step-1 K2 specialised for this cascade (fd_jit.cpp)
    bool jit_tried = false;
    ~fd_cascade_s() {
        fdk::jit_k2_free(jit);
        for (auto& kv : packed) {
            cudaFree(kv.second.d_rec);
            cudaFree(kv.second.d_st);
            cudaFree(kv.second.d_trec);
        }
    }
};
using Packed = fd_cascade_s::Packed;

namespace {

// f3 ("reencoding and combining them into two 16-bit words using simple bitwise
// operations and masks"; reading R13).  binary16 from a float by its bits: exact only if the float's
// exponent is in binary16 range and the dropped fraction bits are zero.  -1 if not representable.
int half_bits_of(float v) {
    uint32_t u;
    std::memcpy(&u, &v, 4);
    const uint32_t sgn = (u >> 16) & 0x8000u, e = (u >> 23) & 255u, m = u & 0x7fffffu;
    if (e == 255u) return -1;                           // inf / nan
    if (e == 0u) return m == 0u ? (int)sgn : -1;        // +-0 (fp32 subnormals are below binary16)
    const int ue = (int)e - 127;                        // unbiased exponent
    if (ue > 15) return -1;
    if (ue >= -14) {                                    // normal binary16: 10 fraction bits
        if (m & 0x1fffu) return -1;
        return (int)(sgn | (uint32_t)(ue + 15) << 10 | (m >> 13));
    }
    // subnormal binary16: value = q * 2^-24 with q = (2^23 + m) * 2^(ue - 23 + 24)
    const int sh = -14 - ue;                            // 1 .. (extra right shift beyond 13)
    if (sh > 10) return -1;
    const uint32_t full = 0x800000u | m;
    if (full & ((1u << (13 + sh)) - 1u)) return -1;
    return (int)(sgn | (full >> (13 + sh)));
}
float half_to_float(uint32_t h) {                        // exact widening
    const uint32_t sgn = (h & 0x8000u) << 16, e = (h >> 10) & 31u, m = h & 1023u;
    uint32_t u;
    if (e == 0u) {
        if (m == 0u) {
            u = sgn;
        } else {                                        // subnormal: normalise
            int ee = -1;
            uint32_t mm = m;
            do {
                ++ee;
                mm <<= 1;
            } while (!(mm & 1024u));
            u = sgn | (uint32_t)(127 - 15 - ee) << 23 | (mm & 1023u) << 13;
        }
    } else {
        u = sgn | (e - 15u + 127u) << 23 | m << 13;
    }
    float v;
    std::memcpy(&v, &u, 4);
    return v;
}

fd_status parse_cascade(const char* text, size_t len, fd_cascade_s* c) {
    std::vector<Line> lines;
    size_t i = 0;
    int no = 0;
    while (i < len) {
        size_t j = i;
        while (j < len && text[j] != '\n') ++j;
        ++no;
        Line L;
        L.no = no;
        std::string cur;
        bool comment = false;
        for (size_t q = i; q < j && !comment; ++q) {
            const char ch = text[q];
            if (ch == '#' && cur.empty() && L.tok.empty()) {
                comment = true;
                break;
            }
            if (ch == ' ' || ch == '\t' || ch == '\r' || ch == '\f' || ch == '\v') {
                if (!cur.empty()) L.tok.push_back(cur), cur.clear();
            } else {
                cur.push_back(ch);
            }
        }
        if (!cur.empty()) L.tok.push_back(cur);
        if (!L.tok.empty()) lines.push_back(std::move(L));
        i = j + 1;
    }
    size_t li = 0;
    auto need = [&](const char* what) -> const Line* {
        if (li >= lines.size()) return nullptr;
        (void)what;
        return &lines[li++];
    };
    const Line* L = need("FDC");
    if (!L || L->tok.size() != 2 || L->tok[0] != "FDC" || L->tok[1] != "1")
        return fail(FD_EFORMAT, "line %d: expected 'FDC 1'", L ? L->no : 0);
    L = need("window");
    if (!L || L->tok.size() != 3 || L->tok[0] != "window" || L->tok[1] != "24" || L->tok[2] != "24")
        return fail(FD_EFORMAT, "line %d: expected 'window 24 24'", L ? L->no : 0);
    L = need("stages");
    if (L && !L->tok.empty() && L->tok[0] == "filter") {      // optional filtering stage (f2, reading R3b)
        if (L->tok.size() == 2 && L->tok[1] == "binomial3")
            c->filter = 1;
        else if (L->tok.size() == 2 && L->tok[1] == "none")
            c->filter = 0;
        else
            return fail(FD_EFORMAT, "line %d: expected 'filter none' or 'filter binomial3'", L->no);
        L = need("stages");
    }
    if (L && !L->tok.empty() && L->tok[0] == "soft") {        // optional soft cascade (f4, reading R8b)
        if (L->tok.size() != 1) return fail(FD_EFORMAT, "line %d: expected 'soft'", L->no);
        c->soft = 1;
        L = need("stages");
    }
    if (L && !L->tok.empty() && L->tok[0] == "compress") {    // optional compressed records (f3, R13)
        if (L->tok.size() != 2 || L->tok[1] != "packed16") return fail(FD_EFORMAT, "line %d: expected 'compress packed16'", L->no);
        c->compressed = 1;
        L = need("stages");
    }
    long ns = 0;
    if (!L || L->tok.size() != 2 || L->tok[0] != "stages" || !parse_int(L->tok[1], &ns) || ns < 1 || ns > 250)
        return fail(FD_EFORMAT, "line %d: expected 'stages N' with 1 <= N <= 250", L ? L->no : 0);
    for (long s = 0; s < ns; ++s) {
        L = need("stage");
        long n = 0;
        HStage st;
        if (!L || L->tok.size() != 3 || L->tok[0] != "stage" || !parse_int(L->tok[1], &n) || n < 1 || n > 65536 ||
            !parse_float(L->tok[2], &st.T, true))
            return fail(FD_EFORMAT, "line %d: expected 'stage n T'", L ? L->no : 0);
        st.first = (int)c->stumps.size();
        st.n = (int)n;
        c->stages.push_back(st);
        for (long j = 0; j < n; ++j) {
            L = need("stump");
            long nr = 0;
            if (!L || L->tok.size() < 2 || L->tok[0] != "stump" || !parse_int(L->tok[1], &nr) || nr < 1 || nr > 3)
                return fail(FD_EFORMAT, "line %d: expected 'stump r ...' with r in 1..3", L ? L->no : 0);
            if ((long)L->tok.size() != 2 + 5 * nr + 3)
                return fail(FD_EFORMAT, "line %d: stump needs %ld rect fields + theta left right", L->no, 5 * nr);
            HStump sp;
            std::memset(&sp, 0, sizeof sp);
            sp.nrect = (int)nr;
            for (long r = 0; r < nr; ++r) {
                long v[5];
                for (int q = 0; q < 5; ++q)
                    if (!parse_int(L->tok[2 + 5 * r + q], &v[q])) return fail(FD_EFORMAT, "line %d: bad rectangle", L->no);
                if (v[0] < 0 || v[1] < 0 || v[2] < 1 || v[3] < 1 || v[0] + v[2] > WIN || v[1] + v[3] > WIN)
                    return fail(FD_EFORMAT, "line %d: rectangle outside the 24x24 window", L->no);
                if (v[4] < -16 || v[4] > 16) return fail(FD_EFORMAT, "line %d: weight outside [-16,16]", L->no);
                for (int q = 0; q < 5; ++q) sp.r[r][q] = (int)v[q];
            }
            const size_t b = 2 + 5 * nr;
            if (!parse_float(L->tok[b], &sp.theta, false) || !parse_float(L->tok[b + 1], &sp.left, false) ||
                !parse_float(L->tok[b + 2], &sp.right, false))
                return fail(FD_EFORMAT, "line %d: expected finite 'theta left right'", L->no);
            c->stumps.push_back(sp);
        }
    }
    if (li != lines.size()) return fail(FD_EFORMAT, "line %d: trailing content", lines[li].no);
    if (c->compressed) {
        // encode each stump into its compressed record, then evaluate what the record says
        c->pk16.assign(c->stumps.size() * FD_PK_WORDS, 0u);
        for (size_t j = 0; j < c->stumps.size(); ++j) {
            HStump& sp = c->stumps[j];
            uint32_t* R = &c->pk16[j * FD_PK_WORDS];
            for (int r = 0; r < sp.nrect; ++r) {
                const int x = sp.r[r][0], y = sp.r[r][1], w = sp.r[r][2], h = sp.r[r][3], wt = sp.r[r][4];
                if (wt < -32 || wt > 31) return fail(FD_EFORMAT, "stump %zu: weight %d outside the packed16 range", j, wt);
                const uint32_t lo = (uint32_t)(x | y << 5 | w << 10), hi = (uint32_t)(h | (wt & 63) << 5);
                R[r] = lo | hi << 16;
                sp.r[r][0] = (int)(R[r] & 31u);
                sp.r[r][1] = (int)((R[r] >> 5) & 31u);
                sp.r[r][2] = (int)((R[r] >> 10) & 31u);
                sp.r[r][3] = (int)((R[r] >> 16) & 31u);
                sp.r[r][4] = (int)(R[r] << 5) >> 26;
            }
            const int th = half_bits_of(sp.theta), lf = half_bits_of(sp.left), rt = half_bits_of(sp.right);
            if (th < 0 || lf < 0 || rt < 0)
                return fail(FD_EFORMAT, "stump %zu: theta/left/right not exactly binary16 (packed16)", j);
            R[3] = (uint32_t)th | (uint32_t)lf << 16;
            R[4] = (uint32_t)rt | (uint32_t)sp.nrect << 16;
            sp.theta = half_to_float(R[3] & 0xffffu);
            sp.left = half_to_float(R[3] >> 16);
            sp.right = half_to_float(R[4] & 0xffffu);
        }
    }
    return FD_OK;
}

// Pack stumps for a tile width TW: each Haar feature is compiled into its distinct
// integral-image corners with integer coefficients (sum_r wt_r * R_r, R = A + D - B - C).
fd_status pack_cascade(fd_cascade_s* c, int TW, Packed* out, bool upload = true) {
    std::vector<uint32_t> rec(c->stumps.size() * REC_WORDS, 0u);
    const size_t ns = c->stumps.size();
    std::vector<uint32_t> trec((size_t)TAIL_REC_WORDS * (ns ? ns : 1), 0u);   // SoA, offsets in TAIL_RP pitch
    for (size_t j = 0; j < c->stumps.size(); ++j) {
        const HStump& s = c->stumps[j];
        int coef[WIN + 1][WIN + 1];
        std::memset(coef, 0, sizeof coef);
        for (int r = 0; r < s.nrect; ++r) {
            const int x = s.r[r][0], y = s.r[r][1], w = s.r[r][2], h = s.r[r][3], wt = s.r[r][4];
            coef[y][x] += wt;
            coef[y][x + w] -= wt;
            coef[y + h][x] -= wt;
            coef[y + h][x + w] += wt;
        }
        uint32_t* R = &rec[j * REC_WORDS];
        int nc = 0;
        for (int y = 0; y <= WIN; ++y)
            for (int x = 0; x <= WIN; ++x)
                if (coef[y][x] != 0) {
                    if (nc == MAX_CORNERS) return fail(FD_EFORMAT, "stump %zu has more than %d corners", j, MAX_CORNERS);
                    const uint32_t off = (uint32_t)(y * TW + x) * 4u;     // byte offset in the smem tile
                    if (off > 0xffffu) return fail(FD_EINVAL, "tile too wide for 16-bit corner offsets");
                    R[4 + nc] = off | ((uint32_t)(coef[y][x] & 0xffff) << 16);
                    trec[(size_t)(4 + nc) * ns + j] = (uint32_t)(y * TAIL_RP + x) | ((uint32_t)(coef[y][x] & 0xffff) << 16);
                    ++nc;
                }
        R[0] = (uint32_t)nc;
        std::memcpy(&R[1], &s.theta, 4);
        std::memcpy(&R[2], &s.left, 4);
        std::memcpy(&R[3], &s.right, 4);
        for (int w = 0; w < 4; ++w) trec[(size_t)w * ns + j] = R[w];
    }
    std::vector<StageDev> st(c->stages.size());
    for (size_t s = 0; s < st.size(); ++s) {
        st[s].first = c->stages[s].first;
        st[s].n = c->stages[s].n;
        st[s].T = c->stages[s].T;
        int mc = 1;
        for (int j = st[s].first; j < st[s].first + st[s].n; ++j)
            mc = (int)rec[(size_t)j * REC_WORDS] > mc ? (int)rec[(size_t)j * REC_WORDS] : mc;
        st[s].mc = mc;
    }
    if (!upload) {
        out->h_rec = std::move(rec);
        out->h_st = std::move(st);
        return FD_OK;
    }
    uint4* d_rec = nullptr;
    StageDev* d_st = nullptr;
    CK(cudaMalloc(&d_rec, rec.size() * 4 + 16));
    CK(cudaMalloc(&d_st, st.size() * sizeof(StageDev)));
    CK(cudaMemcpy(d_rec, rec.data(), rec.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(d_st, st.data(), st.size() * sizeof(StageDev), cudaMemcpyHostToDevice));
    uint32_t* d_trec = nullptr;
    CK(cudaMalloc(&d_trec, trec.size() * 4));
    CK(cudaMemcpy(d_trec, trec.data(), trec.size() * 4, cudaMemcpyHostToDevice));
    out->d_trec = d_trec;
    out->d_rec = d_rec;
    out->d_st = d_st;
    out->h_rec = std::move(rec);
    out->h_st = std::move(st);
    return FD_OK;
}

fd_status get_packed(fd_cascade_s* c, int step, const Packed** out) {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    if (dev != c->device) return fail(FD_EINVAL, "cascade was loaded on device %d, current device is %d", c->device, dev);
    std::lock_guard<std::mutex> lk(c->mu);
    const int TW = tile_w(step);
    auto it = c->packed.find(TW);
    if (it != c->packed.end()) {
        *out = &it->second;
        return FD_OK;
    }
    Packed pk;
    fd_status s = pack_cascade(c, TW, &pk);
    if (s != FD_OK) return s;
    *out = &(c->packed[TW] = std::move(pk));
    return FD_OK;
}

// ------------------------------------------------------------------ tensor maps
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn() {
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeTiledFn>(p);
    });
    return fn;
}

// box_planes: 2 = one TMA brings ii and sqii of a tile (k_cascade), 1 = one plane per TMA
fd_status encode_maps(const PlanDev& p, uint32_t* ws, int step, int box_planes, CUtensorMap* maps) {
    EncodeTiledFn enc = encode_fn();
    if (!enc) return fail(FD_ECUDA, "cuTensorMapEncodeTiled unavailable");
    for (int k = 0; k < p.n_levels; ++k) {
        const LevelDev& L = p.lv[k];
        cuuint64_t dims[4] = {(cuuint64_t)(L.W + 1), (cuuint64_t)(L.H + 1), 2, (cuuint64_t)p.G};
        cuuint64_t strides[3] = {(cuuint64_t)L.P * 4, (cuuint64_t)(L.H + 1) * L.P * 4,
                                 (cuuint64_t)2 * (L.H + 1) * L.P * 4};
        cuuint32_t box[4] = {(cuuint32_t)tile_w(step), (cuuint32_t)tile_h(step), (cuuint32_t)box_planes, 1};
        cuuint32_t es[4] = {1, 1, 1, 1};
        CUresult r = enc(&maps[k], CU_TENSOR_MAP_DATA_TYPE_UINT32, 4, ws + L.ws_off, dims, strides, box, es,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return fail(FD_ECUDA, "cuTensorMapEncodeTiled failed (%d) for level %d", (int)r, k);
    }
    return FD_OK;
}

// f1: one 3-D map per level over the group's level images {x, y, frame}; the box is a tile's
// pixel region (TileGeoF), zero-filled beyond the level
void f1_box(int step, int* bw, int* bh) {
    switch (step) {
        case 1: *bw = TileGeoF<1>::U8W; *bh = TileGeoF<1>::PH; break;
        case 2: *bw = TileGeoF<2>::U8W; *bh = TileGeoF<2>::PH; break;
        case 3: *bw = TileGeoF<3>::U8W; *bh = TileGeoF<3>::PH; break;
        default: *bw = TileGeoF<4>::U8W; *bh = TileGeoF<4>::PH; break;
    }
}

fd_status encode_maps8(const PlanDev& p, uint8_t* ws8, int step, CUtensorMap* maps) {
    EncodeTiledFn enc = encode_fn();
    if (!enc) return fail(FD_ECUDA, "cuTensorMapEncodeTiled unavailable");
    int bw = 0, bh = 0;
    f1_box(step, &bw, &bh);
    for (int k = 0; k < p.n_levels; ++k) {
        const LevelDev& L = p.lv[k];
        cuuint64_t dims[3] = {(cuuint64_t)L.W, (cuuint64_t)L.H, (cuuint64_t)p.G};
        cuuint64_t strides[2] = {(cuuint64_t)L.PB, (cuuint64_t)L.H * L.PB};
        cuuint32_t box[3] = {(cuuint32_t)bw, (cuuint32_t)bh, 1};
        cuuint32_t es[3] = {1, 1, 1};
        CUresult r = enc(&maps[k], CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, ws8 + L.u8_off, dims, strides, box, es,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return fail(FD_ECUDA, "cuTensorMapEncodeTiled (u8) failed (%d) for level %d", (int)r, k);
    }
    return FD_OK;
}

// ------------------------------------------------------------------ kernel accounting
struct Profiler {
    std::mutex mu;
    bool timing = false;
    long long launches[FD_K_COUNT] = {};
    struct Rec {
        int kind;
        cudaEvent_t a, b;
    };
    std::vector<Rec> recs;
    std::vector<cudaEvent_t> pool;
    cudaEvent_t get() {
        if (!pool.empty()) {
            cudaEvent_t e = pool.back();
            pool.pop_back();
            return e;
        }
        cudaEvent_t e = nullptr;
        cudaEventCreate(&e);
        return e;
    }
} g_prof;

// Counts one launch of `kind` (n kernels) and, when timing, brackets it with events.
struct ProfScope {
    int kind;
    cudaStream_t st;
    cudaEvent_t a = nullptr;
    ProfScope(int k, cudaStream_t s, int n = 1) : kind(k), st(s) {
        std::lock_guard<std::mutex> lk(g_prof.mu);
        g_prof.launches[k] += n;
        if (g_prof.timing) {
            a = g_prof.get();
            cudaEventRecord(a, st);
        }
    }
    ~ProfScope() {
        if (!a) return;
        std::lock_guard<std::mutex> lk(g_prof.mu);
        cudaEvent_t b = g_prof.get();
        cudaEventRecord(b, st);
        g_prof.recs.push_back({kind, a, b});
    }
};

#define LAUNCH(kind, st, expr)        \
    do {                              \
        ProfScope ps_((kind), (st));  \
        CK(expr);                     \
    } while (0)

// ------------------------------------------------------------------ workspaces
struct DevBuf {
    void* p = nullptr;
    size_t n = 0;
    ~DevBuf() {
        if (p) cudaFree(p);
    }
    cudaError_t ensure(size_t bytes) {
        if (bytes <= n) return cudaSuccess;
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
        cudaError_t e = cudaMalloc(&p, bytes);
        if (e == cudaSuccess) n = bytes;
        return e;
    }
    template <class T>
    T* as() const {
        return reinterpret_cast<T*>(p);
    }
};

// Per-frame-group buffers of the K1 -> K2 pipeline: integral planes, K1 scratch, tensor maps,
// stage-1 survivor list, tile records and tail queue.  run_groups alternates frame groups
// between two such slots on two streams, so K1 of group g+1 overlaps the latency-bound deep
// stages and tail of group g (different resources: HBM vs issue/latency).
struct PipeSlot {
    DevBuf ws, colbuf, rowbuf, corbuf, lvlbuf, tmaps, tailq, surv, tilerec, tlist;
    // K1 scratch for g frames of plan p
    cudaError_t k1_scratch(const PlanDev& p, int g, K1Scratch* s) {
        cudaError_t e = colbuf.ensure((size_t)g * p.col_frame * 4 + 16);
        if (e == cudaSuccess) e = rowbuf.ensure((size_t)g * p.row_frame * 4 + 16);
        if (e == cudaSuccess) e = corbuf.ensure((size_t)g * p.cor_frame * 8 + 16);
        if (e == cudaSuccess) e = lvlbuf.ensure((size_t)g * p.lvl_frame + 16);
        s->lvl = lvlbuf.as<uint8_t>();
        s->col = colbuf.as<uint32_t>();
        s->row = rowbuf.as<uint32_t>();
        s->cor = corbuf.as<unsigned long long>();
        return e;
    }
};

struct Workspace {
    int device = 0;
    std::mutex mu;                 // one call at a time per (device, stream)
    DevBuf keys, scores, keys2, scores2, cubtmp, ctl, flev, frames, outbuf, group, grpout, lvbuf;
    PipeSlot slot[2];              // pipeline slots (slot 0 also serves fd_integral / fd_build_pyramid)
    cudaStream_t side = nullptr;   // stream of slot 1, forked from / joined to the caller's stream
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    cudaError_t ensure_side() {
        if (side) return cudaSuccess;
        cudaError_t e = cudaStreamCreateWithFlags(&side, cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ev_fork, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ev_join, cudaEventDisableTiming);
        return e;
    }
    cudaError_t k1_scratch(const PlanDev& p, int g, K1Scratch* s) { return slot[0].k1_scratch(p, g, s); }
    unsigned long long* h_pinned = nullptr;     // pinned host word(s) for count read-back
    std::unique_ptr<CascadeParams> params{new CascadeParams()};
    std::unique_ptr<PlanDev> plan{new PlanDev()};
    // host staging of tensor maps + level table (kept alive until the async copies run)
    std::unique_ptr<CUtensorMap[]> h_geo{new CUtensorMap[2 * FD_MAX_LEVELS + (sizeof(LevelDev) * FD_MAX_LEVELS +
                                                                              sizeof(CUtensorMap) - 1) / sizeof(CUtensorMap)]};
    ~Workspace() {
        if (h_pinned) cudaFreeHost(h_pinned);
        if (ev_fork) cudaEventDestroy(ev_fork);
        if (ev_join) cudaEventDestroy(ev_join);
        if (side) cudaStreamDestroy(side);
    }
};

std::mutex g_ws_mu;
std::map<std::pair<int, cudaStream_t>, std::unique_ptr<Workspace>> g_ws;

fd_status get_ws(cudaStream_t st, Workspace** out) {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(g_ws_mu);
    auto& slot = g_ws[{dev, st}];
    if (!slot) {
        slot.reset(new Workspace());
        slot->device = dev;
        CK(cudaMallocHost(&slot->h_pinned, 64));
    }
    *out = slot.get();
    return FD_OK;
}

int env_int(const char* name, int dflt) {
    const char* v = std::getenv(name);
    if (!v || !*v) return dflt;
    return std::atoi(v);
}

fd_status check_frames(const void* d, int n, int W, int H, int pitch) {
    if (!d) return fail(FD_EINVAL, "frames pointer is NULL");
    if (n < 1) return fail(FD_EINVAL, "n must be >= 1");
    if (pitch < W) return fail(FD_EINVAL, "pitch %d < W %d", pitch, W);
    if (n > (1 << 24)) return fail(FD_EINVAL, "at most 2^24 frames per call");
    return FD_OK;
}

// core of fd_detect / fd_detect_depth: the hot path for every frame group.
fd_status run_groups(fd_cascade_s* c, Workspace* w, const uint8_t* d_frames, int n, int W, int H, int pitch,
                     const fd_plan& pl, int step, bool depth, uint8_t* d_depth, float* d_score, long long det_cap,
                     unsigned long long* d_stage_counts, cudaStream_t st,
                     const uint8_t* h_frames = nullptr) {
    if (step > MAX_STEP) return fail(FD_EINVAL, "step %d not supported (1..%d)", step, MAX_STEP);
    const Packed* pk = nullptr;
    fd_status s = get_packed(c, step, &pk);
    if (s != FD_OK) return s;
    // Schedules (all under the same parity tests, tests/test_gpu_parity.py K2_SCHEDULES):
    //   default for hard cascades: K1 -> k_stage1 -> k_deepq, or k_deep1 -> k_tail (below);
    //   FD_F1=1: k_level -> k_f1 -> k_deep1<F1> -> k_tail, no global integral
    //            (FD_F1_SPLIT=0: k_f1 runs every stage);
    //   soft cascades (R8b) and FD_K2_QUEUE=1: K1 -> k_soft (one lane per window, running sums).
    const bool soft = c->soft != 0;
    const bool queue = soft || env_int("FD_K2_QUEUE", 0) != 0;
    const bool f1 = !queue && env_int("FD_F1", 0) != 0;
    // f1 split (default): k_f1 runs stages 0-1, k_deep1 the rest from rebuilt tile integrals
    // (FD_F1_SPLIT=0: k_f1 runs every stage itself)
    const bool f1_split = f1 && env_int("FD_F1_SPLIT", 1) != 0;
    const bool split = !queue && !f1;
    const bool surv = split || f1_split;
    // frames per group: one K2 launch per group.  f1: the group's level images (12.5 MB per 1080p
    // frame) should stay L2-resident between k_level and k_f1 (FD_F1_GROUP_MB, default 64 MB);
    // K1 schedules: the ii/sqii planes (95.8 MB per 1080p frame; FD_GROUP_MB, default 12288 MB).
    // FD_GROUP_FRAMES overrides.  G <= 65535 (tile and tail-queue frame indices are 32-bit, but
    // the tensor maps' frame extent is kept within 16 bits).
    PlanDev one;
    make_plan_dev(pl, W, H, pitch, step, 1, &one);
    const double per_frame = f1 ? (double)one.u8_bytes : (double)one.ws_elems * 4.0;
    int G = env_int("FD_GROUP_FRAMES", 0);
    // (12 GiB: 128 frames of 1080p per group; fewer, larger groups leave fewer drains of the
    // persistent K2 kernels -- deep path 41.0 / 37.1 / 35.0 / 34.0 / 33.5 ms per 512 frames at
    // 16 / 32 / 64 / 128 / 256 frames per group.  The survivor list is sized for the worst case,
    // about as large again as the planes, so both pipeline slots hold ~48 GB at 1080p.)
    const double budget = (double)(f1 ? env_int("FD_F1_GROUP_MB", 64) : env_int("FD_GROUP_MB", 12288)) * 1024.0 * 1024.0;
    if (G <= 0) G = (int)std::min(65535.0, std::floor(budget / (per_frame > 1 ? per_frame : 1)));
    G = std::max(1, std::min(G, std::min(n, 65535)));
    const int ngroups = (n + G - 1) / G;
    // split K2 deep stages: k_deepq (default: warp-autonomous batches over a per-SM pool of tiles)
    // or FD_DEEPQ=0: k_deep1 (a 4-warp CTA per tile, stage-synchronous) + k_tail.  Compressed (f3)
    // cascades default to k_deep1: k_deepq has no lane-group path for the packed records and ran
    // c6q at 970 vs 1890 frames/s; so do groups of fewer than 4 frames (one 1080p frame: 0.55 vs
    // 0.50 ms -- too few tiles per SM for k_deepq's slots to fill)
    const bool deepq = split && env_int("FD_DEEPQ", (c->compressed || G < 4) ? 0 : 1) != 0;
    // FD_DQ_TAIL=s: k_deepq hands every window that enters stage s to k_tail (default 255: never --
    // measured best for c3; stage 9 is close for the OpenCV-shaped c6)
    const int dq_tail = std::max(1, env_int("FD_DQ_TAIL", 255));
    // tail queue (k_tail): FD_TAIL=0 keeps every window inside K2; FD_TAIL_N = windows left in a
    // batch at which it hands them over; FD_TAIL_CAP = queue entries (16 B each) per group
    const bool use_tail = !queue && env_int("FD_TAIL", 1) != 0 && (!deepq || dq_tail < (int)c->stages.size());
    const int tail_cap = use_tail ? std::max(1024, env_int("FD_TAIL_CAP", 1 << 22)) : 0;
    PlanDev& PD = *w->plan;
    make_plan_dev(pl, W, H, pitch, step, G, &PD);
    PD.filter = c->filter;
    PD.aligned4 = ((reinterpret_cast<uintptr_t>(d_frames) | (uintptr_t)pitch) & 3) == 0;
    PD.aligned16 = ((reinterpret_cast<uintptr_t>(d_frames) | (uintptr_t)pitch) & 15) == 0;
    // two pipeline slots on two streams when there is more than one group (FD_PIPE=0: one)
    const int nslots = (ngroups > 1 && env_int("FD_PIPE", 1) != 0) ? 2 : 1;
    K1Scratch k1s[2];
    std::vector<CUtensorMap> maps((size_t)PD.n_levels);
    for (int b = 0; b < nslots; ++b) {
        PipeSlot& sl = w->slot[b];
        if (surv) {
            CK(sl.surv.ensure((size_t)G * (size_t)PD.win_per_frame * 8 + 16));
            CK(sl.tilerec.ensure((size_t)G * PD.tiles_per_frame * 8 + 16));
        }
        if (deepq) CK(sl.tlist.ensure((size_t)G * PD.tiles_per_frame * 16 + 16));
        if (f1) {
            CK(sl.ws.ensure((size_t)PD.u8_bytes + 16));
            s = encode_maps8(PD, sl.ws.as<uint8_t>(), step, maps.data());
        } else {
            CK(sl.ws.ensure((size_t)PD.ws_elems * 4));
            CK(sl.k1_scratch(PD, G, &k1s[b]));
            // tensor maps of this slot's integral planes (global memory, copied in stream order)
            s = encode_maps(PD, sl.ws.as<uint32_t>(), step, 1, maps.data());
        }
        if (s != FD_OK) return s;
        if (use_tail) CK(sl.tailq.ensure((size_t)tail_cap * 16));
        CK(sl.tmaps.ensure(sizeof(CUtensorMap) * FD_MAX_LEVELS));
        std::memcpy(w->h_geo.get() + b * FD_MAX_LEVELS, maps.data(), sizeof(CUtensorMap) * PD.n_levels);
        CK(cudaMemcpyAsync(sl.tmaps.p, w->h_geo.get() + b * FD_MAX_LEVELS, sizeof(CUtensorMap) * PD.n_levels,
                           cudaMemcpyHostToDevice, st));
    }
    // ctl: [0] detection count, [256 B..] per-group K2 tile counters, then per-group tail counts,
    // survivor counts, deep-kernel tile counters and tile-list counts
    CK(w->ctl.ensure(256 + (size_t)ngroups * 20));
    CK(cudaMemsetAsync(w->ctl.p, 0, 256 + (size_t)ngroups * 20, st));
    if (!depth) {
        const size_t cap = (size_t)(det_cap > 0 ? det_cap : 1);
        CK(w->keys.ensure(cap * 8));
        CK(w->scores.ensure(cap * 4));
    }
    CK(w->lvbuf.ensure(sizeof(LevelDev) * FD_MAX_LEVELS));
    char* h_lv = reinterpret_cast<char*>(w->h_geo.get() + 2 * FD_MAX_LEVELS);
    std::memcpy(h_lv, PD.lv, sizeof(LevelDev) * PD.n_levels);
    CK(cudaMemcpyAsync(w->lvbuf.p, h_lv, sizeof(LevelDev) * PD.n_levels, cudaMemcpyHostToDevice, st));
    CascadeParams& P = *w->params;
    P.lv = w->lvbuf.as<LevelDev>();
    P.n_levels = PD.n_levels;
    P.tiles_per_frame = PD.tiles_per_frame;
    P.win_per_frame = PD.win_per_frame;
    P.stumps = pk->d_rec;
    P.stages = pk->d_st;
    P.n_stages = (int)c->stages.size();
    P.n_pstumps = (int)std::min<size_t>(c->stumps.size(), (size_t)PREC_MAX);
    std::memcpy(P.prec, pk->h_rec.data(), (size_t)P.n_pstumps * REC_WORDS * 4);
    P.n_pstages = (int)std::min<size_t>(c->stages.size(), (size_t)PSTAGE_MAX);
    std::memcpy(P.pstages, pk->h_st.data(), (size_t)P.n_pstages * sizeof(StageDev));
    P.det_count = w->ctl.as<unsigned long long>();
    P.det_keys = depth ? nullptr : w->keys.as<unsigned long long>();
    P.det_scores = depth ? nullptr : w->scores.as<float>();
    P.det_cap = depth ? 0 : det_cap;
    P.depth = d_depth;
    P.score = d_score;
    P.stage_counts = d_stage_counts;
    // deep stages with fewer than lane_min windows share lanes among a window's stumps; the
    // group mode covers every window in one pass only while n <= threads / 2
    const int half = k2_threads(step) / 2;
    P.lane_min = std::max(1, std::min(env_int("FD_LANE_MIN", half + 1), half + 1));
    P.tail_cap = tail_cap;
    P.tail_n = std::max(1, env_int("FD_TAIL_N", 8));
    // FD_S_TAIL: every window still alive at this stage is handed to k_tail (default: none, only
    // the FD_TAIL_N rule)
    P.s_tail = deepq ? dq_tail : std::max(1, env_int("FD_S_TAIL", 255));
    // deep stages with at most FD_DEEP_SPLIT windows (<= 64; default 0 = off) run split-stump
    P.split_max = std::max(0, env_int("FD_DEEP_SPLIT", 0));
    // k_stage1 runs stages [0, s0) (FD_S0 = 2, default, or 1); the fused kernels start their
    // deep phase at stage 1
    P.s0 = split ? (env_int("FD_S0", 2) >= 2 ? 2 : 1) : (f1_split ? 2 : 1);
    P.f1 = f1 ? 1 : 0;
    TailParams TP;
    TP.cap = tail_cap;
    TP.step = step;
    TP.lv = P.lv;
    TP.trec = pk->d_trec;
    TP.ns = (int)c->stumps.size();
    // k_tail stages the records of the first deep stages in shared memory (whole stages from
    // stage 1 on, FD_TAIL_SMEM_STUMPS budget, default 256 stumps = 16 KB)
    {
        const int budget = std::max(0, env_int("FD_TAIL_SMEM_STUMPS", 256));
        const int s1 = std::min((int)c->stages.size() - 1, deepq ? dq_tail : 1);
        TP.j0 = c->stages[s1].first;
        int k = s1, m = 0;
        while (k < (int)c->stages.size() && m + c->stages[k].n <= budget) m += c->stages[k++].n;
        TP.nsm = m;
    }
    TP.stages = pk->d_st;
    TP.n_stages = P.n_stages;
    TP.win_per_frame = P.win_per_frame;
    TP.det_count = P.det_count;
    TP.det_keys = P.det_keys;
    TP.det_scores = P.det_scores;
    TP.det_cap = P.det_cap;
    TP.depth = d_depth;
    TP.score = d_score;
    TP.stage_counts = d_stage_counts;
    // step 1: the K2 specialised for this cascade (compiled once, FD_JIT=0 selects the generic kernel)
    JitK2* jit = nullptr;
    if (step == 1 && !queue && env_int("FD_JIT", 1) != 0) {
        std::lock_guard<std::mutex> lk(c->mu);
        if (!c->jit_tried) {
            c->jit_tried = true;
            std::string err;
            c->jit = jit_k2_build(pk->h_rec.data(), pk->h_st.data(), (int)pk->h_st.size(),
                                  c->compressed ? &c->pk16 : nullptr, &err);
            if (!c->jit) return fail(FD_ECUDA, "K2 specialisation: %s", err.c_str());
        }
        jit = c->jit;
    }
    // slot 1's stream starts after everything the caller queued on st so far (and the copies above)
    cudaStream_t sts[2] = {st, st};
    if (nslots == 2) {
        CK(w->ensure_side());
        CK(cudaEventRecord(w->ev_fork, st));
        CK(cudaStreamWaitEvent(w->side, w->ev_fork, 0));
        sts[1] = w->side;
    }
    for (int gi = 0; gi < ngroups; ++gi) {
        // group gi runs on slot gi % nslots; the slot's stream orders it after group gi - nslots,
        // the previous user of the slot's buffers
        const int b = gi % nslots;
        PipeSlot& sl = w->slot[b];
        const cudaStream_t gs = sts[b];
        const int f0 = gi * G, gf = (n - f0) < G ? (n - f0) : G;
        const uint8_t* fr = d_frames + (size_t)f0 * H * pitch;
        const cudaStream_t ks = gs;               // K1's stream
        // host frames (fd_detect_host, fd_detect_group_host): each group's frames are copied on its
        // own slot's stream, so the copy of group g+1 overlaps the kernels of group g
        if (h_frames)
            CK(cudaMemcpyAsync(const_cast<uint8_t*>(fr), h_frames + (size_t)f0 * H * pitch, (size_t)gf * H * pitch,
                               cudaMemcpyHostToDevice, ks));
        if (f1) {
            LAUNCH(FD_K_LEVEL, ks, launch_levels(fr, PD, gf, sl.ws.as<uint8_t>(), ks));
        } else {
            LAUNCH(FD_K_COLSUM, ks, launch_k1_marg(fr, PD, gf, k1s[b], ks));
            {
                ProfScope ps(FD_K_CARRY, ks, 2);
                CK(launch_k1_carry(PD, gf, k1s[b], ks));
            }
            LAUNCH(FD_K_BAND, ks, launch_k1_tiles(fr, PD, gf, k1s[b], sl.ws.as<uint32_t>(), ks));
        }
        P.tmaps = sl.tmaps.as<CUtensorMap>();
        P.tail_q = use_tail ? sl.tailq.as<uint4>() : nullptr;
        P.g_frames = gf;
        P.frame_base = f0;
        P.total_tiles = gf * PD.tiles_per_frame;
        P.tile_counter = reinterpret_cast<unsigned int*>(w->ctl.as<char>() + 256) + gi;
        P.tail_count = reinterpret_cast<unsigned int*>(w->ctl.as<char>() + 256) + ngroups + gi;
        P.surv_count = reinterpret_cast<unsigned int*>(w->ctl.as<char>() + 256) + 2 * ngroups + gi;
        P.deep_counter = reinterpret_cast<unsigned int*>(w->ctl.as<char>() + 256) + 3 * ngroups + gi;
        P.tile_list_count = reinterpret_cast<unsigned int*>(w->ctl.as<char>() + 256) + 4 * ngroups + gi;
        P.tile_list = deepq ? sl.tlist.as<uint4>() : nullptr;
        P.surv = surv ? sl.surv.as<uint2>() : nullptr;
        P.tile_rec = surv ? sl.tilerec.as<uint2>() : nullptr;
        if (queue) {
            LAUNCH(FD_K_CASCADE, gs, launch_soft(P, depth, step, soft, gs));
        } else if (jit) {
            std::string err;
            cudaError_t e;
            {
                ProfScope ps(FD_K_CASCADE, gs);
                e = jit_k2_launch(jit, P, depth, f1 ? JIT_F1 : JIT_STAGE1, gs, &err);
            }
            if (e == cudaSuccess && surv) {
                ProfScope ps(FD_K_DEEP, gs);
                e = jit_k2_launch(jit, P, depth, f1 ? JIT_DEEP1_F1 : (deepq ? JIT_DEEPQ : JIT_DEEP1), gs, &err);
            }
            if (e != cudaSuccess)
                return fail(FD_ECUDA, "specialised K2: %s", err.empty() ? cudaGetErrorString(e) : err.c_str());
        } else if (f1) {
            LAUNCH(FD_K_CASCADE, gs, launch_f1(P, depth, step, gs));
            if (f1_split) LAUNCH(FD_K_DEEP, gs, launch_deep1(P, depth, step, true, gs));
        } else {
            LAUNCH(FD_K_CASCADE, gs, launch_stage1(P, depth, step, gs));
            if (deepq)
                LAUNCH(FD_K_DEEP, gs, launch_deepq(P, depth, step, gs));
            else
                LAUNCH(FD_K_DEEP, gs, launch_deep1(P, depth, step, false, gs));
        }
        if (use_tail) {
            TP.q = P.tail_q;
            TP.ws = f1 ? nullptr : sl.ws.as<uint32_t>();
            TP.lvl8 = f1 ? sl.ws.as<uint8_t>() : nullptr;
            TP.count = P.tail_count;
            TP.frame_base = f0;
            LAUNCH(FD_K_TAIL, gs, launch_tail(TP, depth, gs));
        }
    }
    if (nslots == 2) {       // the caller's stream continues after both slots
        CK(cudaEventRecord(w->ev_join, w->side));
        CK(cudaStreamWaitEvent(st, w->ev_join, 0));
    }
    return FD_OK;
}

fd_status detect_impl(fd_cascade c, const uint8_t* d_frames, int n, int W, int H, int pitch, int min_size, double s,
                      int step, fd_detection* d_out, int64_t capacity, int64_t* n_out, int64_t* d_stage_counts,
                      cudaStream_t st, const uint8_t* h_frames = nullptr) {
    if (!c) return fail(FD_EINVAL, "cascade is NULL");
    if (!n_out) return fail(FD_EINVAL, "n_out is NULL");
    if (capacity < 0) return fail(FD_EINVAL, "capacity < 0");
    if (capacity > 0 && !d_out) return fail(FD_EINVAL, "d_out is NULL");
    fd_status r = check_frames(d_frames, n, W, H, pitch);
    if (r != FD_OK) return r;
    fd_plan pl;
    r = make_plan(W, H, min_size, s, step, &pl);
    if (r != FD_OK) return r;
    Workspace* w = nullptr;
    r = get_ws(st, &w);
    if (r != FD_OK) return r;
    std::lock_guard<std::mutex> lk(w->mu);
    if (pl.n_levels == 0) {
        *n_out = 0;
        return FD_OK;
    }
    const long long cap = capacity > 0 ? capacity : 1;
    r = run_groups(c, w, d_frames, n, W, H, pitch, pl, step, false, nullptr, nullptr, cap,
                   reinterpret_cast<unsigned long long*>(d_stage_counts), st, h_frames);
    if (r != FD_OK) return r;
    CK(cudaMemcpyAsync(w->h_pinned, w->ctl.p, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const long long cnt = (long long)w->h_pinned[0];
    *n_out = cnt;
    if (cnt > capacity) return fail(FD_ECAPACITY, "%lld detections > capacity %lld", cnt, (long long)capacity);
    if (cnt == 0) return FD_OK;
    size_t tb = 0;
    CK(sort_pairs(nullptr, tb, nullptr, nullptr, nullptr, nullptr, cnt, st));
    CK(w->cubtmp.ensure(tb + 16));
    CK(w->keys2.ensure((size_t)cnt * 8));
    CK(w->scores2.ensure((size_t)cnt * 4));
    CK(w->flev.ensure(sizeof(double) * FD_MAX_LEVELS));
    CK(cudaMemcpyAsync(w->flev.p, pl.f, sizeof(double) * FD_MAX_LEVELS, cudaMemcpyHostToDevice, st));
    tb = w->cubtmp.n;
    LAUNCH(FD_K_SORT, st, sort_pairs(w->cubtmp.p, tb, w->keys.as<unsigned long long>(), w->keys2.as<unsigned long long>(),
                  w->scores.as<float>(), w->scores2.as<float>(), cnt, st));
    LAUNCH(FD_K_DETS, st, launch_keys_to_dets(w->keys2.as<unsigned long long>(), w->scores2.as<float>(), cnt, w->flev.as<double>(),
                           (int)c->stages.size(), d_out, st));
    return FD_OK;
}

}  // namespace

// ==================================================================== C ABI
extern "C" {

const char* fd_last_error(void) { return g_err.c_str(); }
int fd_abi_version(void) { return FD_ABI_VERSION; }

fd_status fd_pyramid_plan(int W, int H, int min_size, double scale_factor, int step, fd_plan* out) {
    if (!out) return fail(FD_EINVAL, "out is NULL");
    return make_plan(W, H, min_size, scale_factor, step, out);
}

fd_status fd_load_cascade(const char* text, size_t len, fd_cascade* out) {
    if (!text || !out) return fail(FD_EINVAL, "NULL argument");
    std::unique_ptr<fd_cascade_s> c(new fd_cascade_s());
    fd_status s = parse_cascade(text, len, c.get());
    if (s != FD_OK) return s;
    CK(cudaGetDevice(&c->device));
    const Packed* pk = nullptr;
    s = get_packed(c.get(), 1, &pk);         // upload the step-1 packing now
    if (s != FD_OK) return s;
    *out = c.release();
    return FD_OK;
}

// Diagnostic (not in fd.h's stable set): generate and NVRTC-compile the step-1 K2 specialised
// for a cascade text without touching a device.  FD_OK, or FD_ECUDA with the compiler log.
fd_status fd_debug_jit_compile(const char* text, size_t len, size_t* cubin_bytes) {
    if (!text) return fail(FD_EINVAL, "NULL argument");
    std::unique_ptr<fd_cascade_s> c(new fd_cascade_s());
    fd_status s = parse_cascade(text, len, c.get());
    if (s != FD_OK) return s;
    Packed pk;
    s = pack_cascade(c.get(), tile_w(1), &pk, false);
    if (s != FD_OK) return s;
    std::vector<char> cubin;
    std::vector<std::string> lowered;
    std::string err;
    if (!jit_k2_compile(jit_program(pk.h_rec.data(), pk.h_st.data(), (int)pk.h_st.size(), c->compressed ? &c->pk16 : nullptr),
                        false, &cubin, &lowered, &err))
        return fail(FD_ECUDA, "%s", err.c_str());
    if (cubin_bytes) *cubin_bytes = cubin.size();
    return FD_OK;
}

fd_status fd_free_cascade(fd_cascade c) {
    delete c;
    return FD_OK;
}

fd_status fd_cascade_info(fd_cascade c, int32_t* n_stages, int32_t* n_stumps) {
    if (!c) return fail(FD_EINVAL, "cascade is NULL");
    if (n_stages) *n_stages = (int32_t)c->stages.size();
    if (n_stumps) *n_stumps = (int32_t)c->stumps.size();
    return FD_OK;
}

fd_status fd_build_pyramid(const uint8_t* d_frames, int n, int W, int H, int pitch, int min_size, double scale_factor,
                           uint8_t* d_levels, void* stream) {
    fd_status r = check_frames(d_frames, n, W, H, pitch);
    if (r != FD_OK) return r;
    if (!d_levels) return fail(FD_EINVAL, "d_levels is NULL");
    fd_plan pl;
    r = make_plan(W, H, min_size, scale_factor, 1, &pl);
    if (r != FD_OK) return r;
    if (pl.n_levels == 0) return FD_OK;
    PlanDev p;
    make_plan_dev(pl, W, H, pitch, 1, 1, &p);
    long long off = 0;
    for (int k = 0; k < pl.n_levels; ++k) {      // col_off carries the level byte offset here
        p.lv[k].col_off = off;
        off += (long long)pl.w[k] * pl.h[k];
    }
    LAUNCH(FD_K_PYRAMID, (cudaStream_t)stream, launch_pyramid(d_frames, p, n, d_levels, off, nullptr, (cudaStream_t)stream));
    return FD_OK;
}

fd_status fd_integral(const uint8_t* d_img, int n, int W, int H, int pitch, uint32_t* d_ii, uint64_t* d_sqii,
                      int out_pitch, void* stream) {
    fd_status r = check_frames(d_img, n, W, H, pitch);
    if (r != FD_OK) return r;
    if (W < 1 || H < 1) return fail(FD_EINVAL, "empty image");
    if (!d_ii || !d_sqii) return fail(FD_EINVAL, "output pointer is NULL");
    if (out_pitch < W + 1 || (out_pitch & 3)) return fail(FD_EINVAL, "out_pitch must be >= W+1 and a multiple of 4");
    if ((reinterpret_cast<uintptr_t>(d_ii) & 15) || (reinterpret_cast<uintptr_t>(d_sqii) & 15))
        return fail(FD_EINVAL, "output pointers must be 16-byte aligned");
    cudaStream_t st = (cudaStream_t)stream;
    fd_plan pl;
    std::memset(&pl, 0, sizeof pl);
    pl.n_levels = 1;
    pl.f[0] = 1.0;
    pl.w[0] = W;
    pl.h[0] = H;
    PlanDev p;
    make_plan_dev(pl, W, H, pitch, 1, 1, &p);
    p.aligned4 = ((reinterpret_cast<uintptr_t>(d_img) | (uintptr_t)pitch) & 3) == 0;
    p.aligned16 = ((reinterpret_cast<uintptr_t>(d_img) | (uintptr_t)pitch) & 15) == 0;
    Workspace* w = nullptr;
    r = get_ws(st, &w);
    if (r != FD_OK) return r;
    std::lock_guard<std::mutex> lk(w->mu);
    K1Scratch k1s;
    CK(w->k1_scratch(p, n, &k1s));
    LAUNCH(FD_K_COLSUM, st, launch_k1_marg(d_img, p, n, k1s, st));
    {
        ProfScope ps(FD_K_CARRY, st, 2);
        CK(launch_k1_carry(p, n, k1s, st));
    }
    LAUNCH(FD_K_BAND, st, launch_k1_tiles_canonical(d_img, p, n, k1s, d_ii, d_sqii, out_pitch, st));
    return FD_OK;
}

fd_status fd_detect(fd_cascade c, const uint8_t* d_frames, int n, int W, int H, int pitch, int min_size,
                    double scale_factor, int step, fd_detection* d_out, int64_t capacity, int64_t* n_out, void* stream) {
    return detect_impl(c, d_frames, n, W, H, pitch, min_size, scale_factor, step, d_out, capacity, n_out, nullptr,
                       (cudaStream_t)stream);
}

fd_status fd_detect_ex(fd_cascade c, const uint8_t* d_frames, int n, int W, int H, int pitch, int min_size,
                       double scale_factor, int step, fd_detection* d_out, int64_t capacity, int64_t* n_out,
                       int64_t* d_stage_counts, void* stream) {
    return detect_impl(c, d_frames, n, W, H, pitch, min_size, scale_factor, step, d_out, capacity, n_out,
                       d_stage_counts, (cudaStream_t)stream);
}

fd_status fd_detect_depth(fd_cascade c, const uint8_t* d_frames, int n, int W, int H, int pitch, int min_size,
                          double scale_factor, int step, uint8_t* d_depth, float* d_score, void* stream) {
    if (!c) return fail(FD_EINVAL, "cascade is NULL");
    if (!d_depth || !d_score) return fail(FD_EINVAL, "output pointer is NULL");
    fd_status r = check_frames(d_frames, n, W, H, pitch);
    if (r != FD_OK) return r;
    fd_plan pl;
    r = make_plan(W, H, min_size, scale_factor, step, &pl);
    if (r != FD_OK) return r;
    if (pl.n_levels == 0) return FD_OK;
    cudaStream_t st = (cudaStream_t)stream;
    Workspace* w = nullptr;
    r = get_ws(st, &w);
    if (r != FD_OK) return r;
    std::lock_guard<std::mutex> lk(w->mu);
    return run_groups(c, w, d_frames, n, W, H, pitch, pl, step, true, d_depth, d_score, 0, nullptr, st);
}

fd_status fd_depth_histogram(const uint8_t* d_depth, int n, int W, int H, int min_size, double scale_factor,
                             int step, int n_stages, int64_t* d_hist, void* stream) {
    if (!d_depth || !d_hist) return fail(FD_EINVAL, "depth or histogram pointer is NULL");
    if (n < 1) return fail(FD_EINVAL, "n must be >= 1");
    if (n > 65535) return fail(FD_EINVAL, "at most 65535 frames per call");
    if (n_stages < 1 || n_stages > 254) return fail(FD_EINVAL, "n_stages %d not in [1, 254]", n_stages);
    fd_plan pl;
    fd_status r = make_plan(W, H, min_size, scale_factor, step, &pl);
    if (r != FD_OK) return r;
    if (pl.n_levels == 0) return FD_OK;
    cudaStream_t st = (cudaStream_t)stream;
    Workspace* w = nullptr;
    r = get_ws(st, &w);
    if (r != FD_OK) return r;
    std::lock_guard<std::mutex> lk(w->mu);
    // level window offsets within a frame, and the most levels one 4096-window chunk can span
    long long* h_w0 = reinterpret_cast<long long*>(w->h_geo.get());
    long long acc = 0;
    for (int k = 0; k < pl.n_levels; ++k) {
        h_w0[k] = acc;
        acc += pl.windows[k];
    }
    int max_span = 1;
    for (int k = 0; k < pl.n_levels; ++k) {
        long long reach = h_w0[k] + 4096;
        int j = k;
        while (j + 1 < pl.n_levels && h_w0[j + 1] < reach) ++j;
        max_span = std::max(max_span, j - k + 2);
    }
    max_span = std::min(max_span, pl.n_levels);
    CK(w->flev.ensure(sizeof(double) * FD_MAX_LEVELS));
    CK(cudaMemcpyAsync(w->flev.p, h_w0, sizeof(long long) * pl.n_levels, cudaMemcpyHostToDevice, st));
    {
        ProfScope ps(FD_K_DEPTH_HIST, st);
        CK(launch_depth_hist(d_depth, n, acc, w->flev.as<long long>(), pl.n_levels, n_stages,
                             reinterpret_cast<long long*>(d_hist), max_span, st));
    }
    return FD_OK;
}

fd_status fd_detect_host(fd_cascade c, const uint8_t* h_frames, int n, int W, int H, int pitch, int min_size,
                         double scale_factor, int step, fd_detection* h_out, int64_t capacity, int64_t* n_out,
                         void* stream) {
    if (!h_frames) return fail(FD_EINVAL, "h_frames is NULL");
    if (capacity > 0 && !h_out) return fail(FD_EINVAL, "h_out is NULL");
    fd_status r = check_frames(h_frames, n, W, H, pitch);
    if (r != FD_OK) return r;
    cudaStream_t st = (cudaStream_t)stream;
    Workspace* w = nullptr;
    r = get_ws(st, &w);
    if (r != FD_OK) return r;
    uint8_t* d_fr = nullptr;
    fd_detection* d_out = nullptr;
    {
        std::lock_guard<std::mutex> lk(w->mu);
        CK(w->frames.ensure((size_t)n * H * pitch));
        CK(w->outbuf.ensure((size_t)(capacity > 0 ? capacity : 1) * sizeof(fd_detection)));
        d_fr = w->frames.as<uint8_t>();
        d_out = w->outbuf.as<fd_detection>();
    }
    r = detect_impl(c, d_fr, n, W, H, pitch, min_size, scale_factor, step, d_out, capacity, n_out, nullptr, st, h_frames);
    if (r != FD_OK) return r;
    if (*n_out > 0) CK(cudaMemcpyAsync(h_out, d_out, (size_t)*n_out * sizeof(fd_detection), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    return FD_OK;
}

fd_status fd_group(const fd_detection* d_in, int64_t n, double eyes_thresh, int min_neighbors, fd_detection* d_out,
                   int64_t capacity, int64_t* n_out, void* stream) {
    if (!n_out) return fail(FD_EINVAL, "n_out is NULL");
    if (n < 0 || capacity < 0) return fail(FD_EINVAL, "negative size");
    if (n > 0 && !d_in) return fail(FD_EINVAL, "d_in is NULL");
    if (capacity > 0 && !d_out) return fail(FD_EINVAL, "d_out is NULL");
    if (!(eyes_thresh > 0) || !std::isfinite(eyes_thresh)) return fail(FD_EINVAL, "eyes_thresh must be > 0");
    if (n > (1LL << 31) - 1) return fail(FD_EINVAL, "too many detections");
    if (n == 0) {
        *n_out = 0;
        return FD_OK;
    }
    cudaStream_t st = (cudaStream_t)stream;
    Workspace* w = nullptr;
    fd_status r = get_ws(st, &w);
    if (r != FD_OK) return r;
    std::lock_guard<std::mutex> lk(w->mu);
    CK(w->group.ensure(group_scratch_bytes(n) + 128));
    long long* d_total = reinterpret_cast<long long*>(w->group.as<char>() + w->group.n - 64);
    {
        ProfScope ps(FD_K_GROUP, st, 7);
        CK(launch_group_plan(d_in, n, w->group.p, st));
        CK(launch_group_run(d_in, n, eyes_thresh, min_neighbors < 1 ? 1 : min_neighbors, w->group.p, d_out, capacity,
                            d_total, st));
    }
    CK(cudaMemcpyAsync(w->h_pinned, d_total, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    *n_out = (int64_t)w->h_pinned[0];
    if (*n_out > capacity) return fail(FD_ECAPACITY, "%lld groups > capacity %lld", (long long)*n_out, (long long)capacity);
    return FD_OK;
}

fd_status fd_detect_group_host(fd_cascade c, const uint8_t* h_frames, int n, int W, int H, int pitch, int min_size,
                               double scale_factor, int step, double eyes_thresh, int min_neighbors,
                               fd_detection* h_out, int64_t capacity, int64_t* n_out, int64_t* n_raw, void* stream) {
    if (!h_frames || !n_out) return fail(FD_EINVAL, "NULL argument");
    if (capacity > 0 && !h_out) return fail(FD_EINVAL, "h_out is NULL");
    fd_status r = check_frames(h_frames, n, W, H, pitch);
    if (r != FD_OK) return r;
    cudaStream_t st = (cudaStream_t)stream;
    Workspace* w = nullptr;
    r = get_ws(st, &w);
    if (r != FD_OK) return r;
    uint8_t* d_fr = nullptr;
    fd_detection* d_raw = nullptr;
    int64_t raw_cap = 0;
    {
        std::lock_guard<std::mutex> lk(w->mu);
        CK(w->frames.ensure((size_t)n * H * pitch));
        d_fr = w->frames.as<uint8_t>();
    }
    int64_t cnt = 0;
    for (int attempt = 0; attempt < 2; ++attempt) {
        {
            std::lock_guard<std::mutex> lk(w->mu);
            raw_cap = (int64_t)(w->outbuf.n / sizeof(fd_detection));
            if (raw_cap < 4096) {
                CK(w->outbuf.ensure(4096 * sizeof(fd_detection)));
                raw_cap = 4096;
            }
            d_raw = w->outbuf.as<fd_detection>();
        }
        // the frames are copied group by group inside the first attempt (and are resident for a retry)
        r = detect_impl(c, d_fr, n, W, H, pitch, min_size, scale_factor, step, d_raw, raw_cap, &cnt, nullptr, st,
                        attempt == 0 ? h_frames : nullptr);
        if (r == FD_ECAPACITY && attempt == 0) {
            std::lock_guard<std::mutex> lk(w->mu);
            CK(w->outbuf.ensure((size_t)cnt * sizeof(fd_detection)));
            continue;
        }
        break;
    }
    if (r != FD_OK) return r;
    if (n_raw) *n_raw = cnt;
    fd_detection* d_grp = nullptr;
    {
        std::lock_guard<std::mutex> lk(w->mu);
        CK(w->grpout.ensure((size_t)(cnt > 0 ? cnt : 1) * sizeof(fd_detection)));
        d_grp = w->grpout.as<fd_detection>();
    }
    int64_t ng = 0;
    r = fd_group(d_raw, cnt, eyes_thresh, min_neighbors, d_grp, cnt, &ng, stream);
    if (r != FD_OK) return r;
    *n_out = ng;
    if (ng > capacity) return fail(FD_ECAPACITY, "%lld groups > capacity %lld", (long long)ng, (long long)capacity);
    if (ng > 0) CK(cudaMemcpyAsync(h_out, d_grp, (size_t)ng * sizeof(fd_detection), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    return FD_OK;
}

fd_status fd_profile_reset(int time_kernels) {
    std::lock_guard<std::mutex> lk(g_prof.mu);
    for (auto& r : g_prof.recs) {
        cudaEventSynchronize(r.b);
        g_prof.pool.push_back(r.a);
        g_prof.pool.push_back(r.b);
    }
    g_prof.recs.clear();
    for (int k = 0; k < FD_K_COUNT; ++k) g_prof.launches[k] = 0;
    g_prof.timing = time_kernels != 0;
    return FD_OK;
}

fd_status fd_profile_read(fd_profile* out) {
    if (!out) return fail(FD_EINVAL, "out is NULL");
    std::lock_guard<std::mutex> lk(g_prof.mu);
    std::memset(out, 0, sizeof *out);
    for (int k = 0; k < FD_K_COUNT; ++k) out->launches[k] = g_prof.launches[k];
    for (auto& r : g_prof.recs) {
        CK(cudaEventSynchronize(r.b));
        float ms = 0.f;
        CK(cudaEventElapsedTime(&ms, r.a, r.b));
        out->ms[r.kind] += ms;
    }
    return FD_OK;
}

fd_status fd_release_workspaces(void) {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(g_ws_mu);
    for (auto it = g_ws.begin(); it != g_ws.end();) {
        if (it->first.first == dev) {
            CK(cudaDeviceSynchronize());
            it = g_ws.erase(it);
        } else {
            ++it;
        }
    }
    return FD_OK;
}

}  // extern "C"
