// fd_jit.h -- run-time specialised K2 (fd_jit.cpp); host-only, not part of the C ABI.
#pragma once
#include <string>
#include <vector>

#include "fd_internal.h"

namespace fdk {

struct JitK2;
// kernels of the specialised program: k_stage1 + k_deepq or k_deep1, and the f1 kernels k_f1 +
// k_deep1<F1> (tile integrals rebuilt from level images)
enum { JIT_STAGE1 = 0, JIT_DEEP1 = 1, JIT_F1 = 2, JIT_DEEP1_F1 = 3, JIT_DEEPQ = 4, JIT_KINDS = 5 };
// CUDA source of the generated first stage (stage index `first`..first+n of the packed step-1
// records, REC_WORDS u32 per stump)
std::string jit_stage1_source(const uint32_t* rec_words, int first, int n);
// generated deep stages [1, k_end) (lane-per-window code with immediate corner offsets)
std::string jit_deep_source(const uint32_t* rec_words, const StageDev* st, int k_end, const char* name);
// the whole NVRTC program for a cascade (generated stages + k_cascade.cu)
// pk16: f3 compressed records (FD_PK_WORDS u32 per stump) held in the program's __constant__ bank
// and read by the lane-per-window deep stages, or null
std::string jit_program(const uint32_t* rec_words, const StageDev* st, int n_stages,
                        const std::vector<uint32_t>* pk16 = nullptr);
// NVRTC compile only (no device needed): cubin + lowered names of the JIT_KINDS kernels
bool jit_k2_compile(const std::string& source, bool depth, std::vector<char>* cubin, std::vector<std::string>* lowered,
                    std::string* err);
// specialisation handle for one cascade (code generated now, compiled and loaded on first launch)
JitK2* jit_k2_build(const uint32_t* rec_words, const StageDev* st, int n_stages, const std::vector<uint32_t>* pk16,
                    std::string* err);
// launch (compiling on first use; cudaErrorInvalidSource + *err when NVRTC fails)
cudaError_t jit_k2_launch(JitK2* j, const CascadeParams& p, bool depth, int kind, cudaStream_t st, std::string* err);
void jit_k2_free(JitK2* j);

}  // namespace fdk
