// lp_internal.h -- launcher interface between the liblp host API (liblp.cu) and
// the kernel translation units.  Not part of the public ABI (include/liblp.h).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace lp {

struct NvlsCount;  // lp_device.cuh

// Geometry of one output matrix split into regions.
struct RegionGeom {
  int64_t M, N;        // output rows / cols of this shard
  int64_t ldc;         // row pitch in elements
  int es;              // element size (bytes)
  int RM, RN;          // region shape (elements)
  int64_t P, Q, R;     // region rows, region cols, regions
  int64_t rid_offset;  // global rid of local region 0
};

struct HashInfo {
  int store;      // 0 array, 1 quad CAS, 2 quad lock, 3 cuckoo, 4 cuckoo + lock
  uint32_t cap;   // hash capacity (0 for array; cuckoo: per table)
  uint32_t seed;
  uint32_t max_evict = 0;  // cuckoo eviction bound of the body's inserts (0 = kCuckooMaxEvict)
};

// ---- lp_kernels.cu
cudaError_t launch_cksum_init(void* ck, size_t bytes, const HashInfo& hi, cudaStream_t st);
// Validation + ordered compaction: flags[R], per-CTA failure counts, ascending failed
// list + device count.  With a ticket (a zero-initialised u32 the kernel leaves at 0)
// and R <= kFusedCompactMaxR, the last validate CTA to finish compacts the flags
// itself (1 launch); otherwise a PDL scatter launch follows (2 launches).
// records != null => records mode (no compare, no compaction).
constexpr int64_t kFusedCompactMaxR = 16384;
// re-validation split around a recovery (array table): regions not flagged by the previous validate (beside the
// recovery) and the failed list (after it); mismatches are added to *d_count
cudaError_t launch_validate_skip_count(const RegionGeom& g, uint32_t mask, const void* out, const void* ck,
                                       const uint8_t* flags, unsigned long long* d_count, int sm_count,
                                       cudaStream_t st);
cudaError_t launch_validate_list_count(const RegionGeom& g, uint32_t mask, const void* out, const void* ck,
                                       const int64_t* list, const int64_t* d_n, unsigned long long* d_count,
                                       int sm_count, cudaStream_t st);
cudaError_t launch_validate(const RegionGeom& g, uint32_t mask, const HashInfo& hi, const void* out, const void* ck,
                            uint8_t* flags, uint32_t* records, int sm_count, cudaStream_t st, uint32_t* counts,
                            int64_t* list, int64_t* d_n, uint32_t* ticket = nullptr,
                            const NvlsCount* nv = nullptr);
size_t validate_counts_bytes(const RegionGeom& g, int sm_count);
cudaError_t launch_compact(const RegionGeom& g, const uint8_t* flags, uint32_t* block_counts, int64_t* list,
                           int64_t* d_n, cudaStream_t st);
size_t compact_scratch_bytes(int64_t R);
cudaError_t launch_inject(const RegionGeom& g, uint32_t mask, const HashInfo& hi, void* out, void* ck,
                          const void* stale, const int64_t* rids, int64_t n, uint32_t mode, uint64_t seed,
                          cudaStream_t st);
// ascending list of 128x128 tiles/regions -> recovery tasks of 1-2 entries of the same row band
// (row = (list[i] - off) / div); pairing only when *d_n > min_pair.  tasks[t] = (i << 1) | paired.
// G = 4: tasks of up to four entries (128x64 slices), tasks[t] = (i << 2) | (count - 1).
// The tasks are then ordered by size (largest first) and dealt to the `grid` persistent CTAs of the
// re-execution kernel in alternating direction (CTA i runs positions i, i + grid, ...): an LPT-like static
// schedule.  tasks_tmp: scratch of the same size as tasks.  d_rec (optional) <- *d_n * rec_num / rec_den,
// the regions the re-execution will rewrite (lp_recover_count), so no separate count launch is needed.
cudaError_t launch_pair_tasks(const int64_t* list, const int64_t* d_n, int64_t off, int64_t div, int64_t min_pair,
                              int G, int grid, int32_t* tasks_tmp, int32_t* tasks, int64_t* d_ntasks,
                              int64_t* d_rec, int64_t rec_num, int64_t rec_den, cudaStream_t st);
// cuckoo stores: rebuild T1/T2 with a new seed if the stash is non-empty (no-op otherwise)
cudaError_t launch_cuckoo_rehash(void* ck, cudaStream_t st);
// *dst = *src * num / den on the device (recovered-region count of a list-mode recovery)
cudaError_t launch_scale_count(const int64_t* src, int64_t num, int64_t den, int64_t* dst, cudaStream_t st);
cudaError_t launch_stats(const HashInfo& hi, const void* ck, int64_t* d_stats, cudaStream_t st);
// failed regions -> unique tile ids of an EM x EN tile grid (tile = (p*RM/EM)*(N/EN) + q*RN/EN), ascending
cudaError_t launch_tiles_of_failed(const RegionGeom& g, int EM, int EN, const int64_t* list, const int64_t* d_n,
                                   uint8_t* tile_flags, int64_t T, uint32_t* block_counts, int64_t* tile_list,
                                   int64_t* d_ntiles, cudaStream_t st);

// ---- tmm_simt.cu : SIMT region body (CTA tile == region), paper-shaped
struct TmmArgs {
  const void* A;
  int64_t lda;
  const void* B;
  int64_t ldb;
  void* C;
  int64_t ldc;
  int64_t M, N, K;
  int in_bf16, out_bf16;
  int i32;  // int32 in/out (SIMT body, integer multiply-add)
  int RM, RN;
  uint32_t mask;
  HashInfo hash;
  uint32_t* ck;
  int64_t rid_offset;
  const int64_t* list;  // list mode (recovery) when non-null
  const int64_t* d_n;
  int list_is_tiles;    // list holds 128x128 tile ids (de-duplicated recovery of 32x32 regions)
  int slice64;          // with list_is_tiles: ids are 128x64 slices, a task is 1-4 slices of one row band (N = 64..256)
  void* slice_part;     // 128x128 regions as slices: per-region {2 x CkRecord} partials (workspace)
  uint32_t* slice_cnt;  //   and per-region arrival counters (zero-initialised, self-resetting)
  const int32_t* tasks;  // tcgen05 list mode: paired recovery tasks (launch_pair_tasks), or null
  const int64_t* d_ntasks;
  int force_1cta;       // tcgen05: use the 1-CTA 128x256 kernel even where the CTA-pair kernel applies
  int no_shuffle;       // SIMT: sequential shared-memory reduction (the paper's "no shuffle" ablation)
  int sm_count;
};
bool tmm_simt_supported(int RM, int RN, int in_bf16, int out_bf16);
cudaError_t launch_tmm_simt(const TmmArgs& a, cudaStream_t st);

// ---- tmm_tc.cu : tcgen05 / TMEM / TMA region body (bf16 in)
bool tmm_tc_supported(int64_t M, int64_t N, int64_t K, int RM, int RN, int in_bf16, int64_t lda, int64_t ldb,
                      int64_t ldc, const void* A, const void* B, const void* C);
cudaError_t launch_tmm_tc(const TmmArgs& a, cudaStream_t st, const char** why);
// Listing 7's same-grid check-and-recover on the CTA-pair kernel (M, N % 256 == 0): every CTA validates
// its halves of its pair's tiles, then recomputes in place only the tiles with a failed region;
// *d_rec (zeroed here) counts the failed regions.
bool tmm_tc_check_supported(int64_t M, int64_t N);
// gbits / gbar (workspace, may be null): balanced form -- a cooperative launch whose CTAs publish their failed
// tiles to a global bitmask, pass a grid barrier and deal the failed tiles round robin over all pairs.
cudaError_t launch_tmm_tc_check_recover(const TmmArgs& a, int64_t* d_rec, uint32_t* gbits, uint32_t* gbar,
                                        cudaStream_t st, const char** why);

// ---- tmm_tf32.cu : fp32 in/out via 3xTF32 on tcgen05 (CTA pair)
bool tmm_tf32_supported(int64_t M, int64_t N, int64_t K, int RM, int RN, int in_bf16, int out_bf16, int64_t lda,
                        int64_t ldb, int64_t ldc, const void* A, const void* B, const void* C);
cudaError_t launch_tmm_tf32(const TmmArgs& a, cudaStream_t st, const char** why);

// ---- stencil.cu : 5-point stencil region body
struct StencilArgs {
  const float* in;
  int64_t ldi;
  float* out;
  int64_t ldo;
  int64_t H, W;
  int row_lo, row_span;  // readable input rows, relative to this shard's first row: [row_lo, row_lo + row_span)
                         // = the shard plus its halo rows inside the global domain (zero outside it)
  int RM, RN;
  uint32_t mask;
  HashInfo hash;
  uint32_t* ck;
  int64_t rid_offset;
  const int64_t* list;
  const int64_t* d_n;
  int sm_count;
};
bool stencil_supported(int RM, int RN);
cudaError_t launch_stencil(const StencilArgs& a, cudaStream_t st);
// Listing 7's same-grid check-and-recover (N2): one CTA per region validates and, on
// mismatch, re-executes in place; *d_recovered (zeroed here) counts re-executed regions.
cudaError_t launch_stencil_check_recover(const StencilArgs& a, int64_t* d_recovered, cudaStream_t st);

// ---- spmv.cu : CSR sparse matrix x dense vector region body (N4), regions of RN consecutive rows
struct SpmvArgs {
  const int64_t* row_ptr;  // [m + 1], absolute offsets into col / val (16-B aligned arrays)
  const int32_t* col;
  const float* val;
  const float* x;
  float* y;                // [m]
  int64_t m, n, nnz;       // rows, columns (length of x), stored elements (val / col length)
  int RN;
  uint32_t mask;
  HashInfo hash;
  uint32_t* ck;
  int64_t rid_offset;
  const int64_t* list;
  const int64_t* d_n;
  int no_shuffle;
  int sm_count;
};
bool spmv_supported(int RN);
cudaError_t launch_spmv(const SpmvArgs& a, cudaStream_t st);

// ---- fn_study.cu : false-negative study (N3)
cudaError_t launch_fn_study(uint64_t seed, int64_t trials, int64_t nwords, int mode, int kmax,
                            unsigned long long* counts, uint32_t* dump, int64_t dump_trials, int sm_count,
                            cudaStream_t st);

}  // namespace lp
