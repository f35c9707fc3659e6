// fd_jit.cpp -- run-time specialisation of K2 for one cascade (window step 1).
//
// The first stage runs on every window of every level (94.5% of windows stop there),
// so its code is generated from the cascade and compiled with NVRTC for sm_100a:
//   * every Haar corner becomes an immediate shared-memory offset and an immediate integer
//     coefficient (no record loads, no corner decoding);
//   * a thread owns WPT windows of one column (rows i = 0..WPT-1), so corner (dx, dy) of window i
//     reads tile row dy + i: the stage's corners are grouped by column dx and each distinct
//     (dx, row) value is loaded ONCE per thread and added into every (stump, window)
//     accumulator that uses it (c3's first stage: 536 -> 236 shared loads per thread);
//   * leaf decisions are kept as bits and the leaves are added in stump order at the end, so the
//     fp32 stage sum is the exact sequence of the definition (oracle c7/c8).
// The rest of the kernel is k_cascade.cu itself (embedded at build time, jit_sources.h) compiled
// with -DFD_JIT_STAGE1.  Compiled once per cascade and cached on it.
#include <nvrtc.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "fd_internal.h"
#include "fd_jit.h"
#include "jit_sources.h"

namespace fdk {

// Launch geometry of each kind, fixed when the program is generated (the launch-bound macros
// of the generated source come from the environment at that moment; never re-read at launch).
struct KindGeo {
    int threads = 0;
    size_t smem = 0;
    int grid_per_sm = 0;                          // persistent grid: CTAs per SM (0 = occupancy)
};
struct JitK2 {
    std::string key;                              // generated program (NVRTC source)
    std::vector<uint32_t> pk16;                   // f3 records for the module's __constant__ fd_pk
    KindGeo geo[JIT_KINDS];
    cudaKernel_t kern[2][JIT_KINDS] = {};         // [depth][kind], compiled on first use (g_jit_mu)
    int grid[2][JIT_KINDS] = {};
};

namespace {

constexpr int JIT_STEP = 1;

std::string hexf(uint32_t bits) {
    char b[40];
    std::snprintf(b, sizeof b, "__int_as_float(0x%08x)", bits);
    return b;
}

}  // namespace

std::string jit_stage1_source(const uint32_t* rec_words, int first, int n) {
    constexpr int TW = tile_w(JIT_STEP), WPT = k2_wpt(JIT_STEP);
    struct Use {
        int s, i;
        uint32_t coef;
    };
    std::map<int, std::map<int, std::vector<Use>>> cols;     // dx -> row -> uses
    std::vector<int> last_dx(n, -1);
    for (int s = 0; s < n; ++s) {
        const uint32_t* r = rec_words + (size_t)(first + s) * REC_WORDS;
        const int nc = (int)r[0];
        for (int c = 0; c < nc; ++c) {
            const uint32_t w = r[4 + c];
            const int off = (int)(w & 0xffffu) / 4;
            const uint32_t coef = (uint32_t)((int32_t)w >> 16);
            const int dy = off / TW, dx = off % TW;
            for (int i = 0; i < WPT; ++i) cols[dx][dy + i].push_back({s, i, coef});
            if (dx > last_dx[s]) last_dx[s] = dx;
        }
    }
    std::ostringstream o;
    o << "namespace fdk {\n"
      << "__device__ __forceinline__ void jit_stage1(const uint32_t* __restrict__ T, const float* nf, float* sm) {\n";
    const int nm = (n + 31) / 32;
    for (int s = 0; s < n; ++s)
        for (int i = 0; i < WPT; ++i) o << "  uint32_t a" << s << "_" << i << " = 0u;\n";
    for (int w = 0; w < nm; ++w)
        for (int i = 0; i < WPT; ++i) o << "  uint32_t m" << w << "_" << i << " = 0u;\n";
    for (const auto& col : cols) {
        const int dx = col.first;
        for (const auto& row : col.second) {
            o << "  { const uint32_t v = T[" << row.first * TW + dx << "];";
            for (const Use& u : row.second) {
                o << " a" << u.s << "_" << u.i;
                if (u.coef == 1u)
                    o << " += v;";
                else if (u.coef == 0xffffffffu)
                    o << " -= v;";
                else
                    o << " += v * " << u.coef << "u;";
            }
            o << " }\n";
        }
        for (int s = 0; s < n; ++s) {
            if (last_dx[s] != dx) continue;
            const uint32_t* r = rec_words + (size_t)(first + s) * REC_WORDS;
            for (int i = 0; i < WPT; ++i)
                o << "  if (__int2float_rn((int)a" << s << "_" << i << ") < __fmul_rn(" << hexf(r[1]) << ", nf[" << i
                  << "])) m" << s / 32 << "_" << i << " |= " << (1u << (s % 32)) << "u;\n";
        }
    }
    for (int s = 0; s < n; ++s) {
        const uint32_t* r = rec_words + (size_t)(first + s) * REC_WORDS;
        if (last_dx[s] < 0) {       // a stump without corners: f = 0
            for (int i = 0; i < WPT; ++i)
                o << "  if (0.0f < __fmul_rn(" << hexf(r[1]) << ", nf[" << i << "])) m" << s / 32 << "_" << i
                  << " |= " << (1u << (s % 32)) << "u;\n";
        }
    }
    for (int s = 0; s < n; ++s) {
        const uint32_t* r = rec_words + (size_t)(first + s) * REC_WORDS;
        for (int i = 0; i < WPT; ++i)
            o << "  sm[" << i << "] = __fadd_rn(sm[" << i << "], (m" << s / 32 << "_" << i << " & " << (1u << (s % 32))
              << "u) ? " << hexf(r[2]) << " : " << hexf(r[3]) << ");\n";
    }
    o << "}\n}  // namespace fdk\n";
    return o.str();
}

std::string jit_deep_source(const uint32_t* rec_words, const StageDev* st, int k_end, const char* name) {
    constexpr int TW = tile_w(JIT_STEP);
    std::ostringstream o;
    o << "namespace fdk {\n"
      << "__device__ __forceinline__ float " << name << "(int s, const uint32_t* __restrict__ T, float nf) {\n"
      << "  float sum = 0.0f;\n  switch (s) {\n";
    for (int s = 1; s < k_end; ++s) {
        o << "  case " << s << ":\n";
        for (int j = st[s].first; j < st[s].first + st[s].n; ++j) {
            const uint32_t* r = rec_words + (size_t)j * REC_WORDS;
            const int nc = (int)r[0];
            o << "    { const uint32_t f = 0u";
            for (int c = 0; c < nc; ++c) {
                const uint32_t w = r[4 + c];
                const int off = (int)(w & 0xffffu) / 4;
                const uint32_t coef = (uint32_t)((int32_t)w >> 16);
                (void)TW;
                if (coef == 1u)
                    o << " + T[" << off << "]";
                else if (coef == 0xffffffffu)
                    o << " - T[" << off << "]";
                else
                    o << " + " << coef << "u * T[" << off << "]";
            }
            o << ";\n      sum = __fadd_rn(sum, (__int2float_rn((int)f) < __fmul_rn(" << hexf(r[1]) << ", nf)) ? "
              << hexf(r[2]) << " : " << hexf(r[3]) << "); }\n";
        }
        o << "    break;\n";
    }
    o << "  }\n  return sum;\n}\n}  // namespace fdk\n";
    return o.str();
}

int jit_deep_end(const StageDev* st, int n_stages, const char* env, int budget) {
    if (const char* e = std::getenv(env)) budget = std::atoi(e);   // generated deep stumps (code size bound)
    int k = 1;
    while (k < n_stages && st[k].n <= budget) budget -= st[k++].n;
    return k;
}

static int env_or(const char* name, int dflt) {
    const char* e = std::getenv(name);
    return e && *e ? std::atoi(e) : dflt;
}

// k_deep1 block size of the generated program (FD_K2D_THREADS: 64 or 128)
static int jit_deep_threads() {
    return env_or("FD_K2D_THREADS", FD_K2D_THREADS) <= 64 ? 64 : 128;
}

// k_deepq geometry of the generated program (FD_DQ_SLOTS tile slots, FD_DQ_WARPS warps)
static int jit_dq_slots() {
    const int v = env_or("FD_DQ_SLOTS", FD_DQ_SLOTS);
    return v < 1 ? 1 : (v > 32 ? 32 : v);
}
static int jit_dq_warps() {
    const int v = env_or("FD_DQ_WARPS", FD_DQ_WARPS);
    return v < 1 ? 1 : (v > 32 ? 32 : v);
}


std::string jit_program(const uint32_t* rec_words, const StageDev* st, int n_stages, const std::vector<uint32_t>* pk16) {
    // k_deep1 runs its specialised stages one lane per window even when few windows are left, so
    // it gets the first ~60 stumps; k_deepq's warps each run their own stage, so its generated
    // stages are bounded at ~150 stumps (c3: stages 1-6, ~20 KB of code next to the compact
    // generic loop; measured 43.4 / 42.2 / 41.7 / 41.0 ms per 512 frames at 32 / 60 / 100 / 150)
    const int k_end = jit_deep_end(st, n_stages, "FD_JIT_DEEP_STUMPS", 60);
    const int k_endq = jit_deep_end(st, n_stages, "FD_JIT_DEEPQ_STUMPS", 150);
    std::string pre;
    if (pk16 && !pk16->empty()) {
        // the records are data of this program (its own __constant__ bank); a digest of them in the
        // source keeps cascades with equal generated code from sharing a loaded module
        unsigned long long h = 1469598103934665603ull;
        for (uint32_t w : *pk16) h = (h ^ w) * 1099511628211ull;
        pre = "// packed16 records digest " + std::to_string(h) + "\n#define FD_PACKED_WORDS " +
              std::to_string(pk16->size()) + "\n";
    }
    std::string src = pre + "#define FD_K2D_CTAS " + std::to_string(env_or("FD_K2D_CTAS", FD_K2D_CTAS)) +
                      "\n#define FD_K2D_THREADS " + std::to_string(jit_deep_threads()) +
                      "\n#define FD_F1_CTAS " + std::to_string(env_or("FD_F1_CTAS", FD_F1_CTAS)) +
                      "\n#define FD_DQ_SLOTS " + std::to_string(jit_dq_slots()) +
                      "\n#define FD_DQ_WARPS " + std::to_string(jit_dq_warps()) +
                      "\n#define FD_DQ_GROUP " + std::to_string(env_or("FD_DQ_GROUP", 16)) +
                      "\n#include \"fd_internal.h\"\n" + jit_stage1_source(rec_words, st[0].first, st[0].n) +
                      "#define FD_JIT_STAGE1 1\n";
    // (two functions: one switch over every generated stage bloats k_deep1's code)
    if (k_end > 1) src += jit_deep_source(rec_words, st, k_end, "jit_deep") + "#define FD_JIT_DEEP " + std::to_string(k_end) + "\n";
    if (k_endq > 1)
        src += jit_deep_source(rec_words, st, k_endq, "jit_deepq") + "#define FD_JIT_DEEPQ " + std::to_string(k_endq) + "\n";
    return src + "#include \"k_cascade.cu\"\n";
}

static std::string jit_name(int kind, bool depth) {
    const std::string d = depth ? "true" : "false";
    if (kind == JIT_STAGE1) return "fdk::k_stage1<1, " + d + ">";
    if (kind == JIT_DEEP1) return "fdk::k_deep1<1, " + d + ", false>";
    if (kind == JIT_DEEP1_F1) return "fdk::k_deep1<1, " + d + ", true>";
    if (kind == JIT_DEEPQ) return "fdk::k_deepq<1, " + d + ">";
    return "fdk::k_f1<1, " + d + ">";
}

static KindGeo jit_kind_geo(int kind) {
    KindGeo g;
    g.threads = (kind == JIT_DEEP1 || kind == JIT_DEEP1_F1) ? jit_deep_threads() : k2_threads(JIT_STEP);
    if (kind == JIT_STAGE1) g.smem = TileGeoA<JIT_STEP>::SMEM;
    if (kind == JIT_DEEP1) g.smem = TileGeoD<JIT_STEP, false>::SMEM;
    if (kind == JIT_DEEP1_F1) g.smem = TileGeoD<JIT_STEP, true>::SMEM;
    if (kind == JIT_F1) g.smem = TileGeoF<JIT_STEP>::SMEM;
    if (kind == JIT_DEEPQ) {
        g.threads = jit_dq_warps() * 32;
        g.smem = dq_smem(JIT_STEP, jit_dq_slots(), jit_dq_warps());
    }
    // FD_S1_GRID / FD_DEEP_GRID: cap the persistent grids of k_stage1 / k_deep1 at that many CTAs
    // per SM, so the other pipeline slot's kernels can co-reside
    if (kind == JIT_STAGE1) g.grid_per_sm = env_or("FD_S1_GRID", 0);
    if (kind == JIT_DEEP1 || kind == JIT_DEEP1_F1) g.grid_per_sm = env_or("FD_DEEP_GRID", 0);
    return g;
}

bool jit_k2_compile(const std::string& source, bool depth, std::vector<char>* cubin, std::vector<std::string>* lowered,
                    std::string* err) {
    const char* hdr_src[] = {jit_src_fd_h, jit_src_fd_internal_h, jit_src_k_common_cuh, jit_src_k_cascade_cu,
                             jit_src_k_deepq_cuh};
    const char* hdr_names[] = {"fd.h", "fd_internal.h", "k_common.cuh", "k_cascade.cu", "k_deepq.cuh"};
    nvrtcProgram prog = nullptr;
    if (nvrtcCreateProgram(&prog, source.c_str(), "k_cascade_jit.cu", 5, hdr_src, hdr_names) != NVRTC_SUCCESS) {
        *err = "nvrtcCreateProgram failed";
        return false;
    }
    std::string names[JIT_KINDS];
    for (int k = 0; k < JIT_KINDS; ++k) {
        names[k] = jit_name(k, depth);
        nvrtcAddNameExpression(prog, names[k].c_str());
    }
    const bool packed = source.find("#define FD_PACKED_WORDS") != std::string::npos;
    if (packed) nvrtcAddNameExpression(prog, "&fdk::fd_pk");
    const bool verbose = std::getenv("FD_JIT_VERBOSE") && std::getenv("FD_JIT_VERBOSE")[0] == '1';
    const char* opts[] = {"-arch=sm_100a", "-std=c++17", "--fmad=false", "-lineinfo", "-default-device",
                          "--ptxas-options=-v"};
    const nvrtcResult rc = nvrtcCompileProgram(prog, verbose ? 6 : 5, opts);
    size_t ln = 0;
    nvrtcGetProgramLogSize(prog, &ln);
    std::string log(ln, '\0');
    if (ln) nvrtcGetProgramLog(prog, &log[0]);
    if (verbose) std::fprintf(stderr, "fd: NVRTC K2 (depth=%d): %s\n", (int)depth, log.c_str());
    if (rc != NVRTC_SUCCESS) {
        *err = std::string("NVRTC: ") + nvrtcGetErrorString(rc) + "\n" + log.substr(0, 4000);
        nvrtcDestroyProgram(&prog);
        return false;
    }
    size_t cb = 0;
    nvrtcGetCUBINSize(prog, &cb);
    cubin->resize(cb);
    nvrtcGetCUBIN(prog, cubin->data());
    lowered->assign(JIT_KINDS + 1, std::string());
    for (int k = 0; k < JIT_KINDS; ++k) {
        const char* lw = nullptr;
        nvrtcGetLoweredName(prog, names[k].c_str(), &lw);
        (*lowered)[k] = lw ? lw : "";
    }
    if (packed) {                                 // [JIT_KINDS]: the constant bank of the f3 records
        const char* lw = nullptr;
        nvrtcGetLoweredName(prog, "&fdk::fd_pk", &lw);
        (*lowered)[JIT_KINDS] = lw ? lw : "";
    }
    nvrtcDestroyProgram(&prog);
    return true;
}

JitK2* jit_k2_build(const uint32_t* rec_words, const StageDev* st, int n_stages, const std::vector<uint32_t>* pk16,
                    std::string* err) {
    (void)err;
    std::unique_ptr<JitK2> J(new JitK2());
    J->key = jit_program(rec_words, st, n_stages, pk16);
    if (pk16) J->pk16 = *pk16;
    for (int k = 0; k < JIT_KINDS; ++k) J->geo[k] = jit_kind_geo(k);
    return J.release();
}

namespace {
// process-wide cache: generated program + depth -> loaded kernels (cascades loaded again with
// the same stages reuse the compiled code)
struct Loaded {
    cudaLibrary_t lib = nullptr;
    cudaKernel_t kern[JIT_KINDS] = {};
    int grid[JIT_KINDS] = {};
};
std::mutex g_jit_mu;
std::map<std::pair<std::string, int>, Loaded> g_jit_cache;
}  // namespace

cudaError_t jit_k2_launch(JitK2* J, const CascadeParams& p, bool depth, int kind, cudaStream_t st, std::string* err) {
    const int d = depth ? 1 : 0;
    cudaKernel_t kern = nullptr;
    int kgrid = 0;
    {
        // compile / load once per (program, depth); the handle's kernel table is read and
        // published under the same lock, so concurrent launches on other streams never see a
        // half-filled table
        std::lock_guard<std::mutex> lk(g_jit_mu);
        if (!J->kern[d][0]) {
            Loaded& L = g_jit_cache[{J->key, d}];
            if (!L.kern[0]) {
                std::vector<char> cubin;
                std::vector<std::string> lowered;
                if (!jit_k2_compile(J->key, depth, &cubin, &lowered, err)) {
                    g_jit_cache.erase({J->key, d});
                    return cudaErrorInvalidSource;
                }
                cudaError_t e = cudaLibraryLoadData(&L.lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
                if (e == cudaSuccess && !J->pk16.empty()) {      // f3: fill the module's constant bank once
                    void* dp = nullptr;
                    size_t bytes = 0;
                    e = cudaLibraryGetGlobal(&dp, &bytes, L.lib, lowered[JIT_KINDS].c_str());
                    if (e == cudaSuccess && bytes == J->pk16.size() * 4)
                        e = cudaMemcpy(dp, J->pk16.data(), bytes, cudaMemcpyHostToDevice);
                    else if (e == cudaSuccess)
                        e = cudaErrorInvalidValue;
                }
                int dev = 0, sms = 0;
                if (e == cudaSuccess) e = cudaGetDevice(&dev);
                if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
                for (int k = 0; k < JIT_KINDS && e == cudaSuccess; ++k) {
                    int per = 0;
                    const KindGeo& g = J->geo[k];
                    e = cudaLibraryGetKernel(&L.kern[k], L.lib, lowered[k].c_str());
                    if (e == cudaSuccess)
                        e = cudaKernelSetAttributeForDevice(L.kern[k], cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                            (int)g.smem, dev);
                    if (e == cudaSuccess)
                        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, reinterpret_cast<const void*>(L.kern[k]),
                                                                          g.threads, g.smem);
                    if (g.grid_per_sm > 0 && g.grid_per_sm < per) per = g.grid_per_sm;
                    L.grid[k] = sms * (per > 0 ? per : 1);
                }
                if (e != cudaSuccess) {
                    *err = std::string("JIT kernel load: ") + cudaGetErrorString(e);
                    g_jit_cache.erase({J->key, d});
                    return e;
                }
            }
            for (int k = 0; k < JIT_KINDS; ++k) {
                J->kern[d][k] = L.kern[k];
                J->grid[d][k] = L.grid[k];
            }
        }
        kern = J->kern[d][kind];
        kgrid = J->grid[d][kind];
    }
    const int grid = kgrid < p.total_tiles ? kgrid : p.total_tiles;
    void* args[] = {const_cast<CascadeParams*>(&p)};
    return cudaLaunchKernel(reinterpret_cast<const void*>(kern), dim3(grid), dim3(J->geo[kind].threads), args,
                            J->geo[kind].smem, st);
}

void jit_k2_free(JitK2* J) { delete J; }    // loaded code stays in the process-wide cache

}  // namespace fdk
