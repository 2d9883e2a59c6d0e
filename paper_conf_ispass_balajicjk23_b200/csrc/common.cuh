// Shared internals of libspmv (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <string>

#include "../../include/spmv.h"

namespace spmv {

// Build constants (reading c23; declared in include/spmv.h and DESIGN.md §Plan;
// re-declared independently in oracle/plan.py).
constexpr int TILE_D = 3072;        // stream tile: rows + entries
constexpr int STREAM_MAX = 1024;    // longest row computed inside a stream tile
constexpr int SHORT_MAX = 32;       // canonical order: sequential up to here
constexpr int WARP_MAX = 2048;      // warp-per-row class upper bound (canonical W = 32)
constexpr int CTA_MAX = 16384;      // CTA-per-row class upper bound
constexpr int HUB_CHUNK = 16384;    // merge-path chunk of a hub row
constexpr int CTA_THREADS = 256;    // canonical width of CTA / hub-chunk sums
constexpr int TILE_BUF = TILE_D + STREAM_MAX + 8;  // max entries of a tile (+ alignment slack)
// Scheduling only (never a row's value): plans of at most SMALL_NNZ entries
// and no hub rows run every class in one launch (k_small), where MID rows
// longer than MID_WIDE get a whole CTA (products staged in shared memory).
constexpr int64_t SMALL_NNZ = int64_t(1) << 24;
constexpr int MID_WIDE = 512;

void set_error(const std::string& msg);
const char* get_error();

struct Err {
  spmv_status st;
};

}  // namespace spmv

#define SPMV_CUDA(call)                                                              \
  do {                                                                               \
    cudaError_t e_ = (call);                                                         \
    if (e_ != cudaSuccess) {                                                         \
      spmv::set_error(std::string(#call) + ": " + cudaGetErrorString(e_) + " @" +    \
                      __FILE__ + ":" + std::to_string(__LINE__));                    \
      throw spmv::Err{SPMV_ECUDA};                                                   \
    }                                                                                \
  } while (0)

#define SPMV_FAIL(code, msg)         \
  do {                               \
    spmv::set_error(msg);            \
    throw spmv::Err{code};           \
  } while (0)

#define SPMV_LAUNCH_CHECK() SPMV_CUDA(cudaGetLastError())
