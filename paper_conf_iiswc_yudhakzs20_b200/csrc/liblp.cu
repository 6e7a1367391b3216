// liblp.cu -- host side of the liblp C ABI (include/liblp.h): argument checks,
// table sizing, dispatch of the region bodies / validation / compaction.
//
// lp_config ~ #pragma nvm lpcuda_init(tab, nelems, selem) + the checksum type
// of lpcuda_checksum (L357, L526-538 §VI); lp_run_protected ~ the annotated
// kernel (Listing 6); lp_validate + lp_recover ~ the generated
// check-and-recovery code (Listing 7), in the validate -> compact ->
// re-execute form (Reading R13).
#include <cuda_runtime.h>
#include <stdint.h>

#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>

#include "liblp.h"
#include "lp_device.cuh"
#include "lp_internal.h"

struct lp_ctx {
  lp_config_t cfg;
  uint32_t mask;
  int selem;
  int dev_checked;  // 0 = not yet, 1 = ok
  int sm_count;
  lp::NvlsCount nvls;  // NVLS-fused failed count (lp_attach_nvls_count); mc == nullptr: off
  // lp_recover_revalidate: a side stream for the re-validation of the unflagged regions + fork / join events
  // (created on first use on cfg.device, destroyed by lp_destroy)
  cudaStream_t side = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
};

namespace {

thread_local std::string g_err;

lp_status fail(lp_status s, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
lp_status fail(lp_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

lp_status ok() {
  g_err.clear();
  return LP_OK;
}

lp_status cuda_fail(cudaError_t e, const char* where) {
  return fail(LP_ERR_CUDA, "%s: %s", where, cudaGetErrorString(e));
}

int es_of(int32_t dt) { return dt == LP_BF16 ? 2 : 4; }

bool is_prime(uint64_t n) {
  if (n < 2) return false;
  for (uint64_t d = 2; d * d <= n; ++d)
    if (n % d == 0) return false;
  return true;
}

// quadratic probing: load <= 70% (L267); cuckoo: per-table capacity 1.15 R, total load <= 43.5%
// (L270 bounds the load; 50% is the threshold of two-table cuckoo hashing, where eviction
// cycles become common -- the rehash then has to run often)
uint32_t hash_cap(int64_t R, int store) {
  uint64_t c = store >= LP_STORE_CUCKOO ? (uint64_t)std::ceil((double)R * 1.15) : (uint64_t)std::ceil((double)R / 0.7);
  if (c < 2) c = 2;
  while (!is_prime(c)) ++c;
  return (uint32_t)c;
}

bool aligned16(const void* p) { return (((uintptr_t)p) & 15u) == 0; }

// Checks shared by every call on a workload; fills the region geometry.
lp_status check_wl(const lp_ctx* h, const lp_workload_t* wl, lp::RegionGeom* g) {
  if (!h) return fail(LP_ERR_INVALID_ARG, "null handle");
  if (!wl) return fail(LP_ERR_INVALID_ARG, "null workload");
  if (wl->kind != LP_WL_TMM && wl->kind != LP_WL_STENCIL5 && wl->kind != LP_WL_SPMV)
    return fail(LP_ERR_INVALID_ARG, "unknown workload kind %d", wl->kind);
  if (wl->kind == LP_WL_SPMV) {
    // regions = region_n consecutive rows of y, i.e. y viewed as [m / region_n][region_n]
    const int RM = h->cfg.region_m, RN = h->cfg.region_n;
    if (RM != 1) return fail(LP_ERR_INVALID_ARG, "SPMV regions are 1 x region_n row blocks (region_m must be 1)");
    if (wl->in_dtype != LP_F32 || wl->out_dtype != LP_F32) return fail(LP_ERR_UNSUPPORTED, "SPMV is fp32 -> fp32");
    if (wl->m <= 0 || wl->n <= 0) return fail(LP_ERR_INVALID_ARG, "m and n must be positive");
    if (wl->m % RN) return fail(LP_ERR_INVALID_ARG, "m=%lld not divisible by region_n=%d (Reading R17)", (long long)wl->m, RN);
    if (!lp::spmv_supported(RN)) return fail(LP_ERR_UNSUPPORTED, "SPMV region_n must be a power of two in [4, 16384]");
    if (wl->row_offset < 0 || wl->global_m < wl->row_offset + wl->m || wl->row_offset % RN)
      return fail(LP_ERR_INVALID_ARG, "shard rows [row_offset, row_offset+m) invalid for region_n");
    g->M = wl->m / RN;
    g->N = RN;
    g->ldc = RN;
    g->es = 4;
    g->RM = 1;
    g->RN = RN;
    g->P = g->M;
    g->Q = 1;
    g->R = g->P;
    g->rid_offset = wl->row_offset / RN;
    if (g->rid_offset + g->R > (int64_t)0xFFFFFFFEll && h->cfg.store != LP_STORE_ARRAY)
      return fail(LP_ERR_UNSUPPORTED, "hash stores key on 32-bit rids");
    return LP_OK;
  }
  if (wl->in_dtype < LP_F32 || wl->in_dtype > LP_I32 || wl->out_dtype < LP_F32 || wl->out_dtype > LP_I32)
    return fail(LP_ERR_INVALID_ARG, "unknown dtype");
  if ((wl->in_dtype == LP_I32) != (wl->out_dtype == LP_I32))
    return fail(LP_ERR_UNSUPPORTED, "int32 TMM needs int32 input and output");
  if (wl->m <= 0 || wl->n <= 0) return fail(LP_ERR_INVALID_ARG, "m and n must be positive");
  const int RM = h->cfg.region_m, RN = h->cfg.region_n;
  if (wl->m % RM || wl->n % RN)
    return fail(LP_ERR_INVALID_ARG, "m=%lld, n=%lld not divisible by the region %dx%d (Reading R17)", (long long)wl->m,
                (long long)wl->n, RM, RN);
  const int es = es_of(wl->out_dtype);
  if (wl->ldc < wl->n) return fail(LP_ERR_INVALID_ARG, "ldc < n");
  if ((wl->ldc * es) % 16) return fail(LP_ERR_INVALID_ARG, "ldc*es must be a multiple of 16 bytes");
  if (wl->row_offset < 0 || wl->global_m < wl->row_offset + wl->m)
    return fail(LP_ERR_INVALID_ARG, "shard rows [row_offset, row_offset+m) outside global_m");
  if (wl->row_offset % RM) return fail(LP_ERR_INVALID_ARG, "row_offset not a multiple of region_m");
  if (wl->kind == LP_WL_TMM) {
    if (wl->k <= 0) return fail(LP_ERR_INVALID_ARG, "k must be positive");
  } else {
    if (wl->in_dtype != LP_F32 || wl->out_dtype != LP_F32) return fail(LP_ERR_UNSUPPORTED, "stencil is fp32 -> fp32");
  }
  g->M = wl->m;
  g->N = wl->n;
  g->ldc = wl->ldc;
  g->es = es;
  g->RM = RM;
  g->RN = RN;
  g->P = wl->m / RM;
  g->Q = wl->n / RN;
  g->R = g->P * g->Q;
  g->rid_offset = (wl->row_offset / RM) * g->Q;
  if (g->rid_offset + g->R > (int64_t)0xFFFFFFFEll && h->cfg.store != LP_STORE_ARRAY)
    return fail(LP_ERR_UNSUPPORTED, "hash stores key on 32-bit rids");
  return LP_OK;
}

lp_status check_device(lp_ctx* h) {
  if (h->dev_checked) return LP_OK;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev <= h->cfg.device) {
    cudaGetLastError();
    return fail(LP_ERR_UNSUPPORTED, "no CUDA device %d (%s)", h->cfg.device, cudaGetErrorString(e));
  }
  cudaDeviceProp prop;
  e = cudaGetDeviceProperties(&prop, h->cfg.device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceProperties");
  if (prop.major != 10 || prop.minor != 0)
    return fail(LP_ERR_UNSUPPORTED, "liblp is built for sm_100a; device %d is sm_%d%d", h->cfg.device, prop.major,
                prop.minor);
  h->sm_count = prop.multiProcessorCount;
  h->dev_checked = 1;
  return LP_OK;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

lp::HashInfo hash_info(const lp_ctx* h, const lp::RegionGeom& g) {
  lp::HashInfo hi;
  hi.store = h->cfg.store;
  hi.cap = h->cfg.store == LP_STORE_ARRAY ? 0u : hash_cap(g.R, h->cfg.store);
  hi.seed = h->cfg.hash_seed;
  hi.max_evict = (h->cfg.flags & LP_FLAG_CUCKOO_SHORT_CHAINS) ? 16u : 0u;
  return hi;
}

size_t cksum_bytes(const lp_ctx* h, const lp::RegionGeom& g) {
  if (h->cfg.store == LP_STORE_ARRAY) return (size_t)g.R * 4u * (size_t)h->selem;
  if (h->cfg.store >= LP_STORE_CUCKOO)
    return sizeof(lp::HashHeader) + ((size_t)hash_cap(g.R, h->cfg.store) * 2u + lp::kCuckooStash) * 16u;
  return sizeof(lp::HashHeader) + (size_t)hash_cap(g.R, h->cfg.store) * 4u * (size_t)(1 + h->selem);
}

// Tensor-core tiles covering the output, for recovery de-duplication: 128x128 tiles of
// 32x32 regions (bf16 1-SM list mode) or 256x256 tiles (fp32 3xTF32 CTA-pair list mode).
// 128x64 slices: bf16 list mode of 32x32 regions, two slices of one row band per N = 128 task.
int64_t dedupe_tiles(const lp::RegionGeom& g, int EM, int EN) {
  return (g.M % EM || g.N % EN) ? 0 : (g.M / EM) * (g.N / EN);
}
int64_t dedupe_capacity(const lp::RegionGeom& g) {
  const int64_t a = dedupe_tiles(g, 128, 64), b = dedupe_tiles(g, 128, 128);
  return a > b ? a : b;
}

struct WsLayout {
  size_t flags, counts, tile_flags, tile_counts, tile_list, d_ntiles, tasks, tasks_tmp, d_ntasks, part, cnt, gbits,
      gbar, ticket, total;
};

WsLayout ws_layout(const lp::RegionGeom& g) {
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  const int64_t T = dedupe_capacity(g);
  WsLayout w;
  w.flags = 0;
  w.counts = al((size_t)g.R);
  const size_t counts_bytes = lp::compact_scratch_bytes(g.R) > (size_t)148 * 16 * 4 * 4 ? lp::compact_scratch_bytes(g.R)
                                                                                         : (size_t)148 * 16 * 4 * 4;
  w.tile_flags = w.counts + al(counts_bytes);
  w.tile_counts = w.tile_flags + al((size_t)T);
  w.tile_list = w.tile_counts + al(lp::compact_scratch_bytes(T));
  w.d_ntiles = w.tile_list + al((size_t)T * 8);
  const size_t ntask_bytes = al((size_t)(g.R > T ? g.R : T) * 4);
  w.tasks = w.d_ntiles + 256;                       // recovery tasks, size-sorted + snake order: int32[max(R, T)]
  w.tasks_tmp = w.tasks + ntask_bytes;              // the same tasks in row order (grouping output)
  w.d_ntasks = w.tasks_tmp + ntask_bytes;
  // 128x128 regions recovered as 128x64 slices: per-region slice partials {2 x CkRecord} + arrival counter
  // (zero-initialised, reset by the finishing slice)
  const size_t npart = g.RM == 128 ? (size_t)g.R : 0;
  w.part = w.d_ntasks + 256;
  w.cnt = w.part + al(npart * 32);
  w.gbits = w.cnt + al(npart * 4);                  // balanced check-and-recover: global failed-tile bitmask
  w.gbar = w.gbits + al((size_t)(g.R + 15) / 16 * 4);  //   (2 bits per tile) and its grid-barrier counter
  w.ticket = w.gbar + 256;                          // fused-compaction ticket (u32; zero-initialised, kept at 0)
  w.total = w.ticket + 256;
  return w;
}

size_t workspace_bytes(const lp::RegionGeom& g) { return ws_layout(g).total; }

// Row shard of the stencil: the caller's input pointer is the shard's first row; the halo rows
// above / below exist (and are read) only where the global domain continues (zero padding outside).
void stencil_rows(const lp_workload_t* wl, lp::StencilArgs* a) {
  a->row_lo = wl->row_offset > 0 ? -1 : 0;
  a->row_span = (int)(wl->m + (wl->row_offset + wl->m < wl->global_m ? 1 : 0) - a->row_lo);
}

lp::TmmArgs tmm_args(const lp_ctx* h, const lp_workload_t* wl, const lp::RegionGeom& g, void* out, void* ck,
                     const int64_t* list, const int64_t* d_n) {
  lp::TmmArgs a;
  a.A = wl->a;
  a.lda = wl->lda;
  a.B = wl->b;
  a.ldb = wl->ldb;
  a.C = out;
  a.ldc = wl->ldc;
  a.M = wl->m;
  a.N = wl->n;
  a.K = wl->k;
  a.in_bf16 = wl->in_dtype == LP_BF16;
  a.out_bf16 = wl->out_dtype == LP_BF16;
  a.i32 = wl->in_dtype == LP_I32;
  a.RM = g.RM;
  a.RN = g.RN;
  a.mask = h->mask;
  a.hash = hash_info(h, g);
  a.ck = (uint32_t*)ck;
  a.rid_offset = g.rid_offset;
  a.list = list;
  a.d_n = d_n;
  a.list_is_tiles = 0;
  a.slice64 = 0;
  a.slice_part = nullptr;
  a.slice_cnt = nullptr;
  a.tasks = nullptr;
  a.d_ntasks = nullptr;
  a.force_1cta = (h->cfg.flags & LP_FLAG_TC_1CTA) ? 1 : 0;
  a.no_shuffle = (h->cfg.flags & LP_FLAG_NO_SHUFFLE) ? 1 : 0;
  a.sm_count = h->sm_count;
  return a;
}

// Body dispatch shared by run_protected and recover (list = null for a full run).
lp_status run_body(lp_ctx* h, const lp_workload_t* wl, const lp::RegionGeom& g, void* out, void* ck,
                   const int64_t* list, const int64_t* d_n, cudaStream_t st, void* workspace = nullptr,
                   int64_t* d_rec = nullptr) {
  const lp::HashInfo hi = hash_info(h, g);
  if ((h->cfg.flags & LP_FLAG_NO_SHUFFLE) && wl->kind == LP_WL_STENCIL5)
    return fail(LP_ERR_UNSUPPORTED, "the no-shuffle ablation is not built for the stencil body");
  if (wl->kind == LP_WL_STENCIL5) {
    if (!lp::stencil_supported(g.RM, g.RN)) return fail(LP_ERR_UNSUPPORTED, "stencil supports 128x128 regions");
    if (!wl->a) return fail(LP_ERR_INVALID_ARG, "null stencil input");
    if (!aligned16(wl->a) || !aligned16(out) || (wl->lda * 4) % 16) return fail(LP_ERR_INVALID_ARG, "stencil buffers must be 16-B aligned");
    if (wl->lda < wl->n) return fail(LP_ERR_INVALID_ARG, "lda < n");
    lp::StencilArgs a;
    a.in = (const float*)wl->a;
    a.ldi = wl->lda;
    a.out = (float*)out;
    a.ldo = wl->ldc;
    a.H = wl->m;
    a.W = wl->n;
    stencil_rows(wl, &a);
    a.RM = g.RM;
    a.RN = g.RN;
    a.mask = h->mask;
    a.hash = hi;
    a.ck = (uint32_t*)ck;
    a.rid_offset = g.rid_offset;
    a.list = list;
    a.d_n = d_n;
    a.sm_count = h->sm_count;
    cudaError_t e = lp::launch_stencil(a, st);
    if (e == cudaSuccess && list && d_rec) e = lp::launch_scale_count(d_n, 1, 1, d_rec, st);
    return e == cudaSuccess ? ok() : cuda_fail(e, "stencil launch");
  }
  if (wl->kind == LP_WL_SPMV) {
    if (!wl->a || !wl->b || !wl->row_ptr || !wl->col_idx) return fail(LP_ERR_INVALID_ARG, "null SPMV operand");
    if (!aligned16(out) || !aligned16(wl->a) || !aligned16(wl->col_idx))
      return fail(LP_ERR_INVALID_ARG, "y, values and col_idx must be 16-B aligned");
    if (wl->nnz < 0) return fail(LP_ERR_INVALID_ARG, "negative nnz");
    lp::SpmvArgs a;
    a.row_ptr = wl->row_ptr;
    a.col = wl->col_idx;
    a.val = (const float*)wl->a;
    a.x = (const float*)wl->b;
    a.y = (float*)out;
    a.m = wl->m;
    a.n = wl->n;
    a.nnz = wl->nnz;
    a.RN = g.RN;
    a.mask = h->mask;
    a.hash = hi;
    a.ck = (uint32_t*)ck;
    a.rid_offset = g.rid_offset;
    a.list = list;
    a.d_n = d_n;
    a.no_shuffle = (h->cfg.flags & LP_FLAG_NO_SHUFFLE) ? 1 : 0;
    a.sm_count = h->sm_count;
    cudaError_t e = lp::launch_spmv(a, st);
    if (e == cudaSuccess && list && d_rec) e = lp::launch_scale_count(d_n, 1, 1, d_rec, st);
    return e == cudaSuccess ? ok() : cuda_fail(e, "SPMV launch");
  }
  if (!wl->a || !wl->b) return fail(LP_ERR_INVALID_ARG, "null A or B");
  if (wl->lda < wl->k || wl->ldb < wl->n) return fail(LP_ERR_INVALID_ARG, "lda < k or ldb < n");
  lp::TmmArgs a = tmm_args(h, wl, g, out, ck, list, d_n);
  const bool tc_ok = lp::tmm_tc_supported(wl->m, wl->n, wl->k, g.RM, g.RN, a.in_bf16, wl->lda, wl->ldb, wl->ldc,
                                          wl->a, wl->b, out);
  const bool tf_ok = !a.i32 && lp::tmm_tf32_supported(wl->m, wl->n, wl->k, g.RM, g.RN, a.in_bf16, a.out_bf16,
                                                       wl->lda, wl->ldb, wl->ldc, wl->a, wl->b, out);
  int body = h->cfg.body;
  if (body == LP_BODY_AUTO) body = (tc_ok || tf_ok) && !a.no_shuffle ? LP_BODY_TCGEN05 : LP_BODY_SIMT;
  if (body == LP_BODY_TCGEN05) {
    if (!tc_ok && !tf_ok)
      return fail(LP_ERR_UNSUPPORTED,
                  "tcgen05 body needs 16-B aligned pitches, region 128x128 or 32x32, and either bf16 input with "
                  "m%%128 == 0, n%%128 == 0, k%%64 == 0, or fp32 input/output with m, n %% 256 == 0, k %% 32 == 0");
    const int E = tc_ok ? 128 : 256;  // tile edge of the list-mode kernel
    const bool pairing = !(h->cfg.flags & LP_FLAG_NO_PAIRING);
    // bf16: failed regions become 128x64 slices, grouped 1-4 per N = 64..256 task of one row band.
    //  - 32x32 regions: de-duplicated (1.7x less re-executed work than 128x128 tiles at 5% failed);
    //  - 128x128 regions, with LP_FLAG_RECOVER_SLICES128 (A/B switch; measured slower): two
    //    slices each, so k-slice tasks can fill every SM (205 failed regions on 148 SMs: 410 slices in tasks
    //    of 3 instead of 103 paired 128x256 tasks); a region's two slice partial records are combined
    //    across tasks in the workspace (epi_finish_slice128).  Default: paired 128x128 tiles.
    const bool slices = tc_ok && pairing &&
                        ((g.RM == 32 && !(h->cfg.flags & LP_FLAG_RECOVER_TILE128)) ||
                         (g.RM == 128 && h->mask != 0 && (h->cfg.flags & LP_FLAG_RECOVER_SLICES128)));
    const bool need_dedupe = tf_ok ? true : (g.RM == 32 || slices);
    const int EN = slices ? 64 : E;
    if (list && workspace && need_dedupe && dedupe_tiles(g, E, EN) > 0) {
      // several failed regions may share one tensor-core tile: recompute each tile once
      const WsLayout w = ws_layout(g);
      uint8_t* ws = (uint8_t*)workspace;
      cudaError_t e0 = lp::launch_tiles_of_failed(g, E, EN, list, d_n, ws + w.tile_flags, dedupe_tiles(g, E, EN),
                                                  (uint32_t*)(ws + w.tile_counts), (int64_t*)(ws + w.tile_list),
                                                  (int64_t*)(ws + w.d_ntiles), st);
      if (e0 != cudaSuccess) return cuda_fail(e0, "tile de-duplication");
      a.list = (const int64_t*)(ws + w.tile_list);
      a.d_n = (const int64_t*)(ws + w.d_ntiles);
      a.list_is_tiles = 1;
      a.slice64 = slices ? 1 : 0;
      if (slices && g.RM == 128) {
        a.slice_part = (void*)(ws + w.part);
        a.slice_cnt = (uint32_t*)(ws + w.cnt);
      }
    }
    // regions rewritten = entries of the list the kernel consumes x regions per entry (a de-duplicated
    // tile / slice rewrites every region inside it; without a workspace every listed region recomputes its
    // whole E x E tile): reported by the grouping kernel when it runs, else by a one-thread launch
    const int64_t rec_num = (int64_t)E * (a.list_is_tiles ? EN : E), rec_den = (int64_t)g.RM * g.RN;
    bool rec_done = false;
    if (list && workspace && tc_ok && (a.list_is_tiles || g.RM == 128) && pairing) {
      // pair failed 128x128 tiles of the same row band into 128x256 tasks (or group up to four 128x64 slices)
      const WsLayout w = ws_layout(g);
      uint8_t* ws = (uint8_t*)workspace;
      const int64_t off = a.list_is_tiles ? 0 : g.rid_offset;
      const int64_t div = a.list_is_tiles ? g.N / EN : g.Q;
      const int grid = (int)(g.R < h->sm_count ? g.R : h->sm_count);  // the re-execution grid (launch_cfg)
      cudaError_t e0 = lp::launch_pair_tasks(a.list, a.d_n, off, div, h->sm_count, a.slice64 ? 4 : 2, grid,
                                             (int32_t*)(ws + w.tasks_tmp), (int32_t*)(ws + w.tasks),
                                             (int64_t*)(ws + w.d_ntasks), d_rec, rec_num, rec_den, st);
      rec_done = d_rec != nullptr;
      if (e0 != cudaSuccess) return cuda_fail(e0, "recovery pairing");
      a.tasks = (const int32_t*)(ws + w.tasks);
      a.d_ntasks = (const int64_t*)(ws + w.d_ntasks);
    }
    const char* why = nullptr;
    cudaError_t e = tc_ok ? lp::launch_tmm_tc(a, st, &why) : lp::launch_tmm_tf32(a, st, &why);
    if (e != cudaSuccess) return why ? fail(LP_ERR_CUDA, "tcgen05 launch: %s", why) : cuda_fail(e, "tcgen05 launch");
    if (list && d_rec && !rec_done) {
      e = lp::launch_scale_count(a.d_n, rec_num, rec_den, d_rec, st);
      if (e != cudaSuccess) return cuda_fail(e, "recovered-count launch");
    }
    return ok();
  }
  if (!lp::tmm_simt_supported(g.RM, g.RN, a.in_bf16, a.out_bf16))
    return fail(LP_ERR_UNSUPPORTED, "SIMT body supports 32x32, 64x64 and 128x128 regions");
  if (wl->k % 16) return fail(LP_ERR_UNSUPPORTED, "SIMT body needs k %% 16 == 0");
  cudaError_t e = lp::launch_tmm_simt(a, st);
  if (e == cudaSuccess && list && d_rec) e = lp::launch_scale_count(d_n, 1, 1, d_rec, st);
  return e == cudaSuccess ? ok() : cuda_fail(e, "SIMT TMM launch");
}

// Cuckoo stores: inserts that hit the eviction bound parked their entry in the stash;
// rebuild the tables with a new seed on the device (a no-op launch while the stash is empty).
lp_status cuckoo_rehash(const lp_ctx* h, void* cksum, cudaStream_t st) {
  if (h->cfg.store < LP_STORE_CUCKOO || h->mask == 0) return ok();
  cudaError_t e = lp::launch_cuckoo_rehash(cksum, st);
  return e == cudaSuccess ? ok() : cuda_fail(e, "cuckoo rehash launch");
}

}  // namespace

extern "C" {

int32_t lp_abi_version(void) { return 100; }

const char* lp_last_error(void) { return g_err.c_str(); }

lp_status lp_config(const lp_config_t* cfg, lp_handle* out) {
  if (!cfg || !out) return fail(LP_ERR_INVALID_ARG, "null argument");
  *out = nullptr;
  if (cfg->region_m <= 0 || cfg->region_n <= 0) return fail(LP_ERR_INVALID_ARG, "region shape must be positive");
  if (cfg->cksum & ~7u) return fail(LP_ERR_INVALID_ARG, "unknown checksum bits 0x%x", cfg->cksum);
  if (cfg->store < LP_STORE_ARRAY || cfg->store > LP_STORE_CUCKOO_LOCK) return fail(LP_ERR_INVALID_ARG, "unknown store %d", cfg->store);
  if (cfg->store != LP_STORE_ARRAY && cfg->cksum == 0) return fail(LP_ERR_INVALID_ARG, "a hash store needs a checksum");
  if (cfg->store != LP_STORE_ARRAY && cfg->cksum != LP_CK_MOD && cfg->cksum != (LP_CK_MOD | LP_CK_XOR))
    return fail(LP_ERR_UNSUPPORTED, "hash stores (the ablation) are built for MOD and MOD|XOR records");
  if (cfg->body < LP_BODY_AUTO || cfg->body > LP_BODY_TCGEN05) return fail(LP_ERR_INVALID_ARG, "unknown body %d", cfg->body);
  if (cfg->device < 0) return fail(LP_ERR_INVALID_ARG, "negative device");
  if (cfg->flags & ~(uint32_t)(LP_FLAG_TC_1CTA | LP_FLAG_NO_SHUFFLE | LP_FLAG_NO_PAIRING | LP_FLAG_NO_FUSED_COMPACT |
                                 LP_FLAG_RECOVER_TILE128 | LP_FLAG_CUCKOO_SHORT_CHAINS | LP_FLAG_NVLS_COUNT |
                                 LP_FLAG_RECOVER_SLICES128 | LP_FLAG_TEST_SKIP_REEXEC))
    return fail(LP_ERR_INVALID_ARG, "unknown flags 0x%x", cfg->flags);
  if ((cfg->flags & LP_FLAG_NO_SHUFFLE) && (cfg->body == LP_BODY_TCGEN05 || cfg->cksum != (LP_CK_MOD | LP_CK_XOR)))
    return fail(LP_ERR_UNSUPPORTED, "the no-shuffle ablation is built for the SIMT TMM and SPMV bodies with MOD|XOR");
  if ((int64_t)cfg->region_m * cfg->region_n * 4 > (16ll << 20))
    return fail(LP_ERR_UNSUPPORTED, "regions larger than 16 MiB are not supported");
  lp_ctx* h = new lp_ctx();
  h->cfg = *cfg;
  h->mask = cfg->cksum;
  h->selem = lp::selem_of(cfg->cksum);
  h->dev_checked = 0;
  h->sm_count = 0;
  h->nvls = lp::NvlsCount{nullptr, nullptr, 1};
  *out = h;
  return ok();
}

lp_status lp_destroy(lp_handle h) {
  if (h && h->side) {
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(h->cfg.device);
    cudaEventDestroy(h->ev_fork);
    cudaEventDestroy(h->ev_join);
    cudaStreamDestroy(h->side);
    cudaSetDevice(prev);
  }
  delete h;
  return ok();
}

int32_t lp_device_sm_count(lp_handle h) {
  if (!h) return 0;
  if (check_device(h) != LP_OK) return 0;
  return h->sm_count;
}

lp_status lp_num_regions(lp_handle h, const lp_workload_t* wl, int64_t* r) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (!r) return fail(LP_ERR_INVALID_ARG, "null output");
  *r = g.R;
  return ok();
}

lp_status lp_cksum_bytes(lp_handle h, const lp_workload_t* wl, size_t* bytes) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (!bytes) return fail(LP_ERR_INVALID_ARG, "null output");
  *bytes = cksum_bytes(h, g);
  return ok();
}

lp_status lp_workspace_bytes(lp_handle h, const lp_workload_t* wl, size_t* bytes) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (!bytes) return fail(LP_ERR_INVALID_ARG, "null output");
  *bytes = workspace_bytes(g);
  return ok();
}

lp_status lp_cksum_init(lp_handle h, const lp_workload_t* wl, void* cksum, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (h->mask == 0) return ok();  // unprotected twin: no table
  if (!cksum) return fail(LP_ERR_INVALID_ARG, "null cksum");
  if (!aligned16(cksum)) return fail(LP_ERR_INVALID_ARG, "cksum must be 16-B aligned");
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  cudaError_t e = lp::launch_cksum_init(cksum, cksum_bytes(h, g), hash_info(h, g), (cudaStream_t)stream);
  return e == cudaSuccess ? ok() : cuda_fail(e, "cksum init");
}

lp_status lp_run_protected(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (!out) return fail(LP_ERR_INVALID_ARG, "null out");
  if (!aligned16(out)) return fail(LP_ERR_INVALID_ARG, "out must be 16-B aligned");
  if (h->mask && !cksum) return fail(LP_ERR_INVALID_ARG, "null cksum");
  if (h->mask && !aligned16(cksum)) return fail(LP_ERR_INVALID_ARG, "cksum must be 16-B aligned");
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  if ((s = run_body(h, wl, g, out, cksum, nullptr, nullptr, (cudaStream_t)stream))) return s;
  return cuckoo_rehash(h, cksum, (cudaStream_t)stream);
}

lp_status lp_validate(lp_handle h, const lp_workload_t* wl, const void* out, const void* cksum, int64_t* failed_list,
                      int64_t failed_cap, int64_t* d_n_failed, void* workspace, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (h->mask == 0) return fail(LP_ERR_STATE, "validation needs a checksum (cfg.cksum != 0)");
  if (!out || !cksum || !failed_list || !d_n_failed || !workspace) return fail(LP_ERR_INVALID_ARG, "null argument");
  if (failed_cap < g.R) return fail(LP_ERR_INVALID_ARG, "failed_cap %lld < R %lld", (long long)failed_cap, (long long)g.R);
  if (!aligned16(out) || !aligned16(cksum) || !aligned16(workspace)) return fail(LP_ERR_INVALID_ARG, "buffers must be 16-B aligned");
  if ((g.RN * g.es) % 16) return fail(LP_ERR_INVALID_ARG, "region_n*es must be a multiple of 16 bytes");
  {
    const int cpr = g.RN * g.es / 16;
    if (cpr & (cpr - 1)) return fail(LP_ERR_UNSUPPORTED, "region_n*es/16 must be a power of two");
  }
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  const WsLayout w = ws_layout(g);
  uint8_t* flags = (uint8_t*)workspace + w.flags;
  uint32_t* counts = (uint32_t*)((uint8_t*)workspace + w.counts);
  cudaStream_t st = (cudaStream_t)stream;
  uint32_t* ticket = (h->cfg.flags & LP_FLAG_NO_FUSED_COMPACT) ? nullptr : (uint32_t*)((uint8_t*)workspace + w.ticket);
  cudaError_t e = lp::launch_validate(g, h->mask, hash_info(h, g), out, cksum, flags, nullptr, h->sm_count, st, counts,
                                      failed_list, d_n_failed, ticket, h->nvls.uc ? &h->nvls : nullptr);
  return e == cudaSuccess ? ok() : cuda_fail(e, "validate launch");
}

lp_status lp_recover(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, const int64_t* failed_list,
                     const int64_t* d_n_failed, void* workspace, lp_stream_t stream) {
  return lp_recover_count(h, wl, out, cksum, failed_list, d_n_failed, workspace, nullptr, stream);
}

lp_status lp_recover_count(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, const int64_t* failed_list,
                           const int64_t* d_n_failed, void* workspace, int64_t* d_n_recovered, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (!out || !failed_list || !d_n_failed) return fail(LP_ERR_INVALID_ARG, "null argument");
  if (h->mask && !cksum) return fail(LP_ERR_INVALID_ARG, "null cksum");
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  if (workspace && !aligned16(workspace)) return fail(LP_ERR_INVALID_ARG, "workspace must be 16-B aligned");
  if ((s = run_body(h, wl, g, out, cksum, failed_list, d_n_failed, (cudaStream_t)stream, workspace, d_n_recovered)))
    return s;
  return cuckoo_rehash(h, cksum, (cudaStream_t)stream);
}

// True when the list-mode recovery writes exactly the listed regions (and their records): stencil, SpMV, the SIMT
// TMM, and the tcgen05 bf16 TMM with 128x128 regions (tile = region).  The tcgen05 bodies with regions smaller
// than their recovery tile (bf16 32x32 in 128x64 slices, fp32 3xTF32 in 256x256 tiles) also rewrite the clean
// regions sharing a tile (identical bits), which a re-validation running beside the recovery would race.
bool recovery_writes_only_listed(const lp_ctx* h, const lp_workload_t* wl, const lp::RegionGeom& g, const void* out) {
  if (wl->kind != LP_WL_TMM) return true;
  const bool i32 = wl->in_dtype == LP_I32, in_bf16 = wl->in_dtype == LP_BF16, out_bf16 = wl->out_dtype == LP_BF16;
  const bool tc_ok = lp::tmm_tc_supported(wl->m, wl->n, wl->k, g.RM, g.RN, in_bf16, wl->lda, wl->ldb, wl->ldc, wl->a,
                                          wl->b, out);
  const bool tf_ok = !i32 && lp::tmm_tf32_supported(wl->m, wl->n, wl->k, g.RM, g.RN, in_bf16, out_bf16, wl->lda,
                                                     wl->ldb, wl->ldc, wl->a, wl->b, out);
  const bool no_shuffle = (h->cfg.flags & LP_FLAG_NO_SHUFFLE) != 0;
  int body = h->cfg.body;
  if (body == LP_BODY_AUTO) body = (tc_ok || tf_ok) && !no_shuffle ? LP_BODY_TCGEN05 : LP_BODY_SIMT;
  if (body != LP_BODY_TCGEN05) return true;
  return tc_ok && g.RM == 128 && g.RN == 128;
}

lp_status lp_recover_revalidate(lp_handle h, const lp_workload_t* wl, void* out, void* cksum,
                                const int64_t* failed_list, const int64_t* d_n_failed, void* workspace,
                                int64_t* d_n_after, int64_t* d_n_recovered, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (!out || !cksum || !failed_list || !d_n_failed || !workspace || !d_n_after)
    return fail(LP_ERR_INVALID_ARG, "null argument");
  if (h->mask == 0 || h->cfg.store != LP_STORE_ARRAY)
    return fail(LP_ERR_UNSUPPORTED, "recover + split re-validation needs checksums in the array store (hash-store "
                                    "inserts move other entries: use lp_recover then lp_validate)");
  if (!aligned16(workspace)) return fail(LP_ERR_INVALID_ARG, "workspace must be 16-B aligned");
  if (!recovery_writes_only_listed(h, wl, g, out))
    return fail(LP_ERR_UNSUPPORTED, "this body's recovery rewrites whole tensor-core tiles (regions smaller than the "
                                    "tile): use lp_recover then lp_validate");
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  cudaError_t e = cudaSuccess;
  if (!h->side) {
    // the side stream gets the LOWEST priority: the recovery's CTAs (a persistent grid that needs whole SMs)
    // are dispatched first, the re-validation fills the SMs and cycles they leave
    int lo_prio = 0, hi_prio = 0;
    cudaDeviceGetStreamPriorityRange(&lo_prio, &hi_prio);
    if ((e = cudaStreamCreateWithPriority(&h->side, cudaStreamNonBlocking, lo_prio)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_fork, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&h->ev_join, cudaEventDisableTiming)) != cudaSuccess)
      return cuda_fail(e, "side stream / events");
  }
  cudaStream_t st = (cudaStream_t)stream;
  const WsLayout w = ws_layout(g);
  const uint8_t* flags = (const uint8_t*)workspace + w.flags;   // the previous lp_validate's per-region flags
  unsigned long long* cnt = reinterpret_cast<unsigned long long*>(d_n_after);
  if ((e = cudaMemsetAsync(d_n_after, 0, sizeof(int64_t), st)) != cudaSuccess) return cuda_fail(e, "memset");
  // fork: the unflagged regions are re-validated on the side stream while the main stream recovers the flagged
  // ones (the recovery is submitted first; the side stream depends only on the work before the fork)
  if ((e = cudaEventRecord(h->ev_fork, st)) != cudaSuccess || (e = cudaStreamWaitEvent(h->side, h->ev_fork, 0)) != cudaSuccess)
    return cuda_fail(e, "fork");
  if (!(h->cfg.flags & LP_FLAG_TEST_SKIP_REEXEC) &&
      (s = run_body(h, wl, g, out, cksum, failed_list, d_n_failed, st, workspace, d_n_recovered)))
    return s;
  if ((e = lp::launch_validate_skip_count(g, h->mask, out, cksum, flags, cnt, h->sm_count, h->side)) != cudaSuccess)
    return cuda_fail(e, "re-validate (unflagged regions)");
  if ((e = cudaEventRecord(h->ev_join, h->side)) != cudaSuccess) return cuda_fail(e, "join record");
  if ((e = cudaStreamWaitEvent(st, h->ev_join, 0)) != cudaSuccess) return cuda_fail(e, "join");
  e = lp::launch_validate_list_count(g, h->mask, out, cksum, failed_list, d_n_failed, cnt, h->sm_count, st);
  return e == cudaSuccess ? ok() : cuda_fail(e, "re-validate (recovered regions)");
}

lp_status lp_check_recover(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, int64_t* d_n_recovered,
                           lp_stream_t stream) {
  return lp_check_recover_ws(h, wl, out, cksum, d_n_recovered, nullptr, stream);
}

lp_status lp_check_recover_ws(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, int64_t* d_n_recovered,
                              void* workspace, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (wl->kind == LP_WL_SPMV) return fail(LP_ERR_UNSUPPORTED, "same-grid check-and-recover: STENCIL5 and TMM only");
  if (h->mask == 0) return fail(LP_ERR_STATE, "check-and-recover needs a checksum (cfg.cksum != 0)");
  if (!out || !cksum || !d_n_recovered || !wl->a) return fail(LP_ERR_INVALID_ARG, "null argument");
  if (wl->kind == LP_WL_TMM) {
    if (!wl->b) return fail(LP_ERR_INVALID_ARG, "null B");
    if (wl->lda < wl->k || wl->ldb < wl->n) return fail(LP_ERR_INVALID_ARG, "lda < k or ldb < n");
    if (h->cfg.body == LP_BODY_SIMT || (h->cfg.flags & (LP_FLAG_TC_1CTA | LP_FLAG_NO_SHUFFLE)) ||
        !lp::tmm_tc_supported(wl->m, wl->n, wl->k, g.RM, g.RN, wl->in_dtype == LP_BF16, wl->lda, wl->ldb, wl->ldc,
                              wl->a, wl->b, out) ||
        !lp::tmm_tc_check_supported(wl->m, wl->n))
      return fail(LP_ERR_UNSUPPORTED,
                  "TMM check-and-recover runs on the tcgen05 CTA-pair body: bf16 input, m, n %% 256 == 0, k %% 64 == 0, "
                  "128x128 or 32x32 regions");
    if (!aligned16(cksum)) return fail(LP_ERR_INVALID_ARG, "cksum must be 16-B aligned");
    if ((s = check_device(h))) return s;
    DeviceGuard dg(h->cfg.device);
    const lp::TmmArgs a = tmm_args(h, wl, g, out, cksum, nullptr, nullptr);
    const char* why = nullptr;
    if (workspace && !aligned16(workspace)) return fail(LP_ERR_INVALID_ARG, "workspace must be 16-B aligned");
    const WsLayout w = ws_layout(g);
    uint32_t* gbits = workspace ? (uint32_t*)((uint8_t*)workspace + w.gbits) : nullptr;
    uint32_t* gbar = workspace ? (uint32_t*)((uint8_t*)workspace + w.gbar) : nullptr;
    cudaError_t e = lp::launch_tmm_tc_check_recover(a, d_n_recovered, gbits, gbar, (cudaStream_t)stream, &why);
    if (e != cudaSuccess) return why ? fail(LP_ERR_UNSUPPORTED, "check-and-recover: %s", why) : cuda_fail(e, "check-and-recover launch");
    if ((s = cuckoo_rehash(h, cksum, (cudaStream_t)stream))) return s;
    return ok();
  }
  if (!lp::stencil_supported(g.RM, g.RN)) return fail(LP_ERR_UNSUPPORTED, "stencil supports 128x128 regions");
  if (!aligned16(wl->a) || !aligned16(out) || (wl->lda * 4) % 16) return fail(LP_ERR_INVALID_ARG, "stencil buffers must be 16-B aligned");
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  lp::StencilArgs a;
  a.in = (const float*)wl->a;
  a.ldi = wl->lda;
  a.out = (float*)out;
  a.ldo = wl->ldc;
  a.H = wl->m;
  a.W = wl->n;
  stencil_rows(wl, &a);
  a.RM = g.RM;
  a.RN = g.RN;
  a.mask = h->mask;
  a.hash = hash_info(h, g);
  a.ck = (uint32_t*)cksum;
  a.rid_offset = g.rid_offset;
  a.list = nullptr;
  a.d_n = nullptr;
  a.sm_count = h->sm_count;
  cudaError_t e = lp::launch_stencil_check_recover(a, d_n_recovered, (cudaStream_t)stream);
  return e == cudaSuccess ? ok() : cuda_fail(e, "check-and-recover launch");
}

lp_status lp_attach_nvls_count(lp_handle h, void* mc_counter, void* uc_counter, int32_t world_size) {
  if (!h) return fail(LP_ERR_INVALID_ARG, "null handle");
  if (!mc_counter && !uc_counter) {
    h->nvls = lp::NvlsCount{nullptr, nullptr, 1};
    return ok();
  }
  if (!(h->cfg.flags & LP_FLAG_NVLS_COUNT)) return fail(LP_ERR_STATE, "lp_config_t.flags lacks LP_FLAG_NVLS_COUNT");
  if (!mc_counter || !uc_counter) return fail(LP_ERR_INVALID_ARG, "both the multicast and the unicast address are needed");
  if ((((uintptr_t)mc_counter) & 63u) || (((uintptr_t)uc_counter) & 63u))
    return fail(LP_ERR_INVALID_ARG, "counter buffers must be 64-B aligned");
  if (world_size < 1) return fail(LP_ERR_INVALID_ARG, "world_size must be >= 1");
  if (mc_counter == uc_counter && world_size != 1)
    return fail(LP_ERR_INVALID_ARG, "mc == uc (single-GPU emulation) needs world_size == 1");
  h->nvls = lp::NvlsCount{(unsigned long long*)mc_counter, (unsigned long long*)uc_counter, world_size};
  return ok();
}

lp_status lp_region_checksums(lp_handle h, const lp_workload_t* wl, const void* out, uint32_t* records,
                              lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (h->mask == 0) return fail(LP_ERR_STATE, "records need a checksum (cfg.cksum != 0)");
  if (!out || !records) return fail(LP_ERR_INVALID_ARG, "null argument");
  if (!aligned16(out)) return fail(LP_ERR_INVALID_ARG, "out must be 16-B aligned");
  {
    const int cpr = g.RN * g.es / 16;
    if ((g.RN * g.es) % 16 || (cpr & (cpr - 1))) return fail(LP_ERR_UNSUPPORTED, "region_n*es/16 must be a power of two");
  }
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  cudaError_t e = lp::launch_validate(g, h->mask, hash_info(h, g), out, nullptr, nullptr, records, h->sm_count,
                                      (cudaStream_t)stream, nullptr, nullptr, nullptr);
  return e == cudaSuccess ? ok() : cuda_fail(e, "records launch");
}

lp_status lp_inject(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, const void* stale,
                    const int64_t* rids, int64_t n, uint32_t mode, uint64_t seed, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (mode > LP_INJ_STALE_RECORD) return fail(LP_ERR_INVALID_ARG, "unknown injection mode %u", mode);
  if (n < 0 || n > g.R) return fail(LP_ERR_INVALID_ARG, "n outside [0, R]");
  if (n == 0) return ok();
  if (!out || !rids) return fail(LP_ERR_INVALID_ARG, "null argument");
  if ((mode == LP_INJ_STALE_WORDS || mode == LP_INJ_STALE_REGION) && !stale)
    return fail(LP_ERR_INVALID_ARG, "stale image required for this mode");
  if (mode == LP_INJ_STALE_RECORD && (h->mask == 0 || !cksum)) return fail(LP_ERR_INVALID_ARG, "STALE_RECORD needs a table");
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  cudaError_t e = lp::launch_inject(g, h->mask, hash_info(h, g), out, cksum, stale, rids, n, mode, seed,
                                    (cudaStream_t)stream);
  return e == cudaSuccess ? ok() : cuda_fail(e, "inject launch");
}

lp_status lp_stats(lp_handle h, const lp_workload_t* wl, const void* cksum, int64_t* d_stats, lp_stream_t stream) {
  lp::RegionGeom g;
  lp_status s = check_wl(h, wl, &g);
  if (s) return s;
  if (!d_stats) return fail(LP_ERR_INVALID_ARG, "null d_stats");
  if (h->cfg.store != LP_STORE_ARRAY && !cksum) return fail(LP_ERR_INVALID_ARG, "null cksum");
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  cudaError_t e = lp::launch_stats(hash_info(h, g), cksum, d_stats, (cudaStream_t)stream);
  return e == cudaSuccess ? ok() : cuda_fail(e, "stats launch");
}

lp_status lp_fn_study(lp_handle h, uint32_t model, int32_t kmax, int64_t region_words, uint64_t seed, int64_t trials,
                      uint64_t* d_counts, uint32_t* dump, int64_t dump_trials, lp_stream_t stream) {
  if (!h || !d_counts) return fail(LP_ERR_INVALID_ARG, "null argument");
  if (model > 3 || kmax < 1 || kmax > 8 || region_words < 2 || trials < 0 || dump_trials < 0)
    return fail(LP_ERR_INVALID_ARG, "model 0..3, kmax 1..8, region_words >= 2");
  if (dump_trials > 0 && !dump) return fail(LP_ERR_INVALID_ARG, "null dump");
  lp_status s;
  if ((s = check_device(h))) return s;
  DeviceGuard dg(h->cfg.device);
  cudaError_t e = lp::launch_fn_study(seed, trials, region_words, (int)model, kmax, (unsigned long long*)d_counts,
                                      dump, dump_trials, h->sm_count, (cudaStream_t)stream);
  return e == cudaSuccess ? ok() : cuda_fail(e, "fn_study launch");
}

}  // extern "C"
