// Plan object (owned device buffers) — internal.
#pragma once
#include <vector>

#include "common.cuh"

// 16-byte stream-tile descriptor (built by the plan, read by k_panel):
// packed = cnt (entries streamed, 14 bits) | (rend - r0) << 14 | last_long << 28
struct TileDesc {
  int64_t e0;
  int32_t r0;
  uint32_t packed;
};

// a BIG_CHUNK-aligned tile of a big row in the key scratch of spmv_permute:
// row start o, row length L, tile start q within the row
struct BigTile {
  int64_t o, L, q;
};

struct spmv_plan_s {
  int device = 0;
  spmv_opts_t opts{};
  cudaStream_t s = nullptr;  // internal stream for the synchronous plan phase

  // global problem
  int64_t n = 0, nnz = 0;
  bool off64 = false;  // local row_ptr stored as int64 (global nnz >= 2^31)

  // borrowed input (valid until spmv_permute completes)
  const int32_t* A_rp32 = nullptr;
  const int64_t* A_rp64 = nullptr;
  const int32_t* A_col = nullptr;
  const float* A_val = nullptr;

  // owned: permutation
  int32_t* d_perm = nullptr;  // perm[old] = new (identity if none given)
  int32_t* d_inv = nullptr;   // inv[new] = old
  int64_t* d_srcA = nullptr;  // [nrows] start in A of each local row of B

  // partition
  int world = 1, rank = 0;
  std::vector<int64_t> part;  // b_0..b_world (global rows)
  int64_t row_begin = 0, row_end = 0, nrows = 0, nnz_local = 0, nnz_before = 0;
  int64_t x_len = 0, x_stride = 0, y_offset = 0;

  // owned: local block of B
  void* d_rp = nullptr;        // int32 or int64 [nrows+1], local offsets
  int32_t* d_col = nullptr;    // [nnz_local + pad]
  float* d_val = nullptr;      // [nnz_local + pad]

  // bins
  int64_t K = 0, n_cta = 0, n_hub = 0, n_chunks = 0, H = 0, max_hub_len = 0;
  int64_t H_nnz = 0;  // entries of B whose column is in the hot prefix [0, H)
  int32_t* d_tiles = nullptr;      // [K+1]
  TileDesc* d_desc = nullptr;      // [K]
  int64_t n_warp = 0;
  int32_t* d_warp_rows = nullptr;  // [n_warp] k_panel: last-in-tile rows, 1024 < L <= 2048
  int64_t n_mid = 0;
  int32_t* d_mid_rows = nullptr;   // [n_mid] k_lane: all rows with 32 < L <= 2048
  int64_t n_mid_wide = 0;          // small plans: MID-list positions q of rows with L > MID_WIDE
  int32_t* d_mid_wide = nullptr;   // [n_mid_wide] (k_small gives each a CTA)
  int32_t* d_cta_rows = nullptr;   // [n_cta]
  int32_t* d_hub_rows = nullptr;   // [n_hub]
  int32_t* d_hub_choff = nullptr;  // [n_hub+1] first chunk of each hub row
  int32_t* d_chunk_row = nullptr;  // [n_chunks]
  int32_t* d_chunk_idx = nullptr;  // [n_chunks]

  // exec scratch
  double* d_chunk_part = nullptr;  // [n_chunks]
  double* d_chunk_part4 = nullptr; // [4 n_chunks] spmv_exec_spmm4 (allocated on first use)


  // COO form of B (spmv_exec_coo; built on first use): row index per entry and
  // per-tile pieces of rows that cross a 2048-entry tile boundary
  int64_t coo_tiles = 0;
  int32_t* d_coo_row = nullptr;    // [nnz_local + 8]
  int32_t* d_coo_trow = nullptr;   // [2 coo_tiles] first / last row of each tile
  double* d_coo_tpart = nullptr;   // [2 coo_tiles] fp64 pieces (first / last row)
  uint8_t* d_coo_tflag = nullptr;  // [coo_tiles]
  bool coo_memset = false;         // a run of > 32 empty rows: memset y, no in-kernel zeroing
  double* d_ss = nullptr;          // [4] iterate scalars
  double* d_ss_part = nullptr;     // [nrows / 16384 + 2] segment sums of the norm (Σy² over y)
  float* d_u = nullptr;            // iterate ping-pong [x_len]

  // permute-phase sort buckets (ascending local rows)
  int32_t* s1 = nullptr; int64_t n1 = 0;        // 32 < L <= 128
  int32_t* s2 = nullptr; int64_t n2 = 0;        // 128 < L <= 1024
  int32_t* s3 = nullptr; int64_t n3 = 0;        // 1024 < L <= 4096
  int32_t* big = nullptr; int64_t nbig = 0;     // L > 4096 (chunk sort + merges)
  int64_t* boff = nullptr; int64_t big_total = 0, big_max = 0;
  BigTile* btile = nullptr; int64_t nbtile = 0;  // BIG_CHUNK-aligned tiles of the big rows
  int32_t* longrows = nullptr; int64_t nlong = 0;  // L > STREAM_MAX

  // exec concurrency: the row-class kernels other than the short-row kernel
  // run on two plan-owned streams forked from / joined to the caller's stream
  cudaStream_t aux[2] = {nullptr, nullptr};
  cudaEvent_t ev_fork = nullptr, ev_join[2] = {nullptr, nullptr};
  bool conc = false, conc_init = false;
  bool stream_ef = false;  // k_lane streams col/val with L2::evict_first (plan decision)
  bool lane_pred = false;  // k_lane gathers x only for a row's own slots (plan decision)
  int64_t lane_nnz = 0;    // entries in short rows (1 <= L <= SHORT_MAX)
  int64_t lane_waste = 0;  // foreign chunk slots k_lane reads in short rows spanning >= 2 chunks
  bool val_nonfinite = false;  // B holds an Inf / NaN value: lane kernels mask values too

  // power iteration across ranks (iterate.cu): collective backend
  // (spmv_set_coll, else NCCL on opts.nccl_comm) and the peer next-x buffers
  // of SPMV_EXCHANGE_PEER (spmv_set_peers), [j * world + k]
  spmv_coll_t coll{};
  bool has_coll = false;
  std::vector<float*> peers;

  // state
  bool permuted = false;
  int64_t l2_window_bytes = 0;
  bool win_alternating = false;  // set by spmv_iterate: x alternates between two buffers
  bool l2_limit_raised = false;   // cudaLimitPersistingL2CacheSize raised by set_window
  size_t l2_limit_before = 0;
  const void* win_ptr = nullptr;
  cudaStream_t win_stream[3] = {nullptr, nullptr, nullptr};
};

namespace spmv {
// x layout of a multi-rank plan (opts.x_layout): padded slices of M floats per
// rank, or (default) B's own row ids, x_len = n
inline bool padded(const spmv_plan_s* p) {
  return p->world > 1 && p->opts.x_layout == SPMV_XLAYOUT_PADDED;
}
void plan_build(spmv_plan_s* p, const spmv_csr_t* A, const int32_t* perm);
void rabbitpp_gpu(const spmv_csr_t* A, const int32_t* perm_rabbit, const int32_t* comm,
                  int32_t* perm_out, cudaStream_t s);
void plan_permute(spmv_plan_s* p, cudaStream_t s);
void plan_free(spmv_plan_s* p);
void permute_vec(spmv_plan_s* p, const float* in, float* out, int inverse, cudaStream_t s);
void pad_vec(spmv_plan_s* p, const float* in, float* out, int to_padded, cudaStream_t s);
void exec(spmv_plan_s* p, const float* x, float* y, const double* ss_in, double* ss_out,
          cudaStream_t s, float* const* bcast = nullptr, int nbcast = 0);
void iterate(spmv_plan_s* p, float* x, int iters, double* lambda, cudaStream_t s);
void iterate_finish(const float* u, float* x, int64_t n, const double* ss, double* lambda,
                    cudaStream_t s);
int exec_launches(const spmv_plan_s* p, bool ss);
void exec_spmm4(spmv_plan_s* p, const float* X, float* Y, cudaStream_t s);
int spmm4_launches(const spmv_plan_s* p);
int lane_ef_mode(const spmv_plan_s* p);
int lane_pred_mode(const spmv_plan_s* p);
void exec_coo(spmv_plan_s* p, const float* x, float* y, cudaStream_t s);
void export_coo_rows(spmv_plan_s* p, int32_t* rows, cudaStream_t s);
void coo_free(spmv_plan_s* p);
void scale_vec(const float* u, float* x, int64_t n, const double* ss, cudaStream_t s);
}  // namespace spmv
