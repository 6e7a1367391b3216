// tc_common.cuh -- tcgen05 / TMEM building blocks and the LP epilogue shared by the
// tensor-core region bodies (tmm_tc.cu: bf16; tmm_tf32.cu: fp32 via 3xTF32).
#pragma once

#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "lp_device.cuh"
#include "lp_ptx.cuh"

namespace lp {
namespace {

constexpr int kBM = 128;      // tile rows per CTA (TMEM lanes)
constexpr int kEpiWarp0 = 2;

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tc_mma(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                       uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}

#define LP_TMEM_LD32(taddr, r)                                                                                       \
  asm volatile(                                                                                                      \
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,"   \
      "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"                                                 \
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),  \
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),       \
        "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),      \
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])                    \
      : "r"(taddr))

__device__ __forceinline__ void tc_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

#define LP_TMEM_ST32(taddr, r)                                                                                       \
  asm volatile(                                                                                                      \
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,"  \
      "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};"                                                    \
      ::"r"(taddr), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),           \
        "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]),      \
        "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]),    \
        "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])                                       \
      : "memory")

__device__ __forceinline__ void tc_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// Shared-memory matrix descriptor (sm_100 UMMA): start>>4 [0,14), LBO>>4 [16,30),
// SBO>>4 [32,46), version 1 [46,48), layout SWIZZLE_128B = 2 at [61,64).
__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

__device__ __forceinline__ void named_bar_epi() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

// C tile stores: evict-first (streaming) so the output does not push the A / B panels the next tiles
// re-read out of L2 (LP_C_STORE_CS=0 builds plain stores for A/B runs)
#ifndef LP_C_STORE_CS
#define LP_C_STORE_CS 1
#endif
__device__ __forceinline__ void st_c16(uint4* p, uint4 v) {
#if LP_C_STORE_CS
  __stcs(p, v);
#else
  *p = v;
#endif
}

// Tile order: groups of LP_TILE_GROUP M-blocks, M fastest inside a group (L2 reuse of B panels).  8: a
// wave of 74 CTA-pair tiles spans 8 A panels x ~9 B panels (the smallest footprint; 16 and 4 measured
// 1.23 / 1.56 GB of DRAM reads per 8192^3 body vs 1.05 GB, profiles/r02/ab_raster.txt).
#ifndef LP_TILE_GROUP
#define LP_TILE_GROUP 8
#endif
__device__ __forceinline__ void tile_coords_g(int64_t t, int64_t num_m, int64_t num_n, int64_t G, int64_t& mb,
                                              int64_t& nb) {
  const int64_t per_group = G * num_n;
  const int64_t g = t / per_group, w = t - g * per_group;
  const int64_t rows = (num_m - g * G) < G ? (num_m - g * G) : G;
  mb = g * G + w % rows;
  nb = w / rows;
}
__device__ __forceinline__ void tile_coords(int64_t t, int64_t num_m, int64_t num_n, int64_t& mb, int64_t& nb) {
  constexpr int64_t G = LP_TILE_GROUP;
  const int64_t per_group = G * num_n;
  const int64_t g = t / per_group, w = t - g * per_group;
  const int64_t rows = (num_m - g * G) < G ? (num_m - g * G) : G;
  mb = g * G + w % rows;
  nb = w / rows;
}

struct TileSrc {
  int64_t num_m, num_n;       // tile grid
  const int64_t* list;        // list mode: failed global rids
  const int64_t* d_n;
  int64_t rid_offset;
  int64_t Qr;                 // regions per output row band
  int reg;                    // region edge (32 or 128)
  int list_is_tiles;          // list holds tile ids (already de-duplicated)
  const int32_t* tasks;       // paired list mode: (list index << 1) | paired (launch_pair_tasks)
  const int64_t* d_ntasks;
  int64_t n128;               // 128-column tiles per row (tile-id decoding)
  int slice64;                // list holds 128x64 slice ids (n64 per row); a task is 1-4 slices (slices())
  int64_t n64;
  int l2_prefetch;            // list mode: k-blocks of the task's operands prefetched into L2 ahead of the ring
  CkRecord* part;             // 128x128 regions as slices: per-region {2 x CkRecord} partials
  uint32_t* cnt;              //   per-region arrival counters (epi_finish_slice128)
  __device__ __forceinline__ int64_t count() const {
    return tasks ? *d_ntasks : (list ? *d_n : num_m * num_n);
  }
  // a list entry (128x128 tile id, or global rid of a 128x128 region) -> 128-row block, 128-col block
  __device__ __forceinline__ void entry128(int64_t e, int64_t& mb, int64_t& cb) const {
    if (list_is_tiles) {
      mb = e / n128;
      cb = e - mb * n128;
    } else {
      const int64_t rid = e - rid_offset;
      mb = rid / Qr;
      cb = rid - mb * Qr;
    }
  }
  // Columns of tile t as two 128-column halves: [n_lo, n_lo+128) and, if has_hi,
  // [n_hi, n_hi+128).  Full runs with BN = 256: contiguous halves; paired list
  // mode: two failed tiles of the same row band (B gathered from two panels).
  template <int BN>
  __device__ __forceinline__ void cols(int64_t t, int64_t& mb, int64_t& n_lo, int64_t& n_hi, bool& has_hi) const {
    if (tasks) {
      const int32_t w = tasks[t];
      const int64_t i = w >> 1;
      int64_t cb;
      entry128(list[i], mb, cb);
      n_lo = cb * 128;
      has_hi = (w & 1) != 0;
      n_hi = n_lo;
      if (has_hi) {
        int64_t mb1, cb1;
        entry128(list[i + 1], mb1, cb1);
        n_hi = cb1 * 128;
      }
      return;
    }
    int64_t nb;
    coords<BN>(t, mb, nb);
    n_lo = nb * BN;
    n_hi = n_lo + 128;
    has_hi = BN == 256;
  }
  // Slice task t (slice64): 1-4 128x64 slices of one row band, first columns nc[0..cnt);
  // B chunk c is staged from slice c's column panel and lands in accumulator columns [64c, 64c+64).
  __device__ __forceinline__ void slices(int64_t t, int64_t& mb, int& cnt, int64_t (&nc)[4]) const {
    const int32_t w = tasks[t];
    const int64_t i = w >> 2;
    cnt = (w & 3) + 1;
    mb = list[i] / n64;
#pragma unroll
    for (int c = 0; c < 4; ++c) nc[c] = c < cnt ? (list[i + c] - mb * n64) * 64 : 0;
  }
  template <int BN>
  __device__ __forceinline__ void coords(int64_t t, int64_t& mb, int64_t& nb) const {
    if (!list) {
      tile_coords(t, num_m, num_n, mb, nb);
      return;
    }
    if (list_is_tiles) {
      mb = list[t] / num_n;
      nb = list[t] - mb * num_n;
      return;
    }
    const int64_t rid = list[t] - rid_offset;
    const int64_t p = rid / Qr, q = rid - p * Qr;
    mb = p * reg / kBM;
    nb = q * reg / BN;
  }
};

// ---------------------------------------------------------------------------- epilogue pieces
// Store one 128-row x BN-column accumulator (this warp's 32 TMEM lanes) to C and
// fold the exact stored words into the LP checksum (L192).  m128 = index of the
// 128-row block of C, n0 = first column.  32x32 regions are finished here (one
// warp-wide redux per checksum, Listing 4); 128x128 regions leave one partial
// per warp in srec for epi_finish_128.
//
// add_prev / final_pass (fp32 output only; used by the K-chunked 3xTF32 body):
// add_prev = C already holds the sum of the previous K chunks -> store C + chunk
// (IEEE round-to-nearest fp32 add); the checksum is folded on the final pass only.
template <typename OutT, uint32_t MASK, int REG, int BN, int STORE>
__device__ __forceinline__ void epi_store(uint32_t t_row, OutT* __restrict__ C, int64_t ldc, int64_t m128, int64_t n0,
                                          int wq, int lane, CkRecord* srec_acc, uint32_t* __restrict__ ck, int64_t Qr,
                                          int64_t rid_offset, bool add_prev = false, bool final_pass = true) {
  constexpr int ES = (int)sizeof(OutT);
  constexpr int NCH = BN / 32;
  const int row_in_tile = wq * 32 + lane;
  OutT* crow = C + (m128 * kBM + row_in_tile) * ldc + n0;
  CkPartial<MASK> part;
  uint4 pf[8];  // prefetched previous partial sums (add_prev only)
  if constexpr (ES == 4) {
    if (add_prev) {
      const uint4* src = reinterpret_cast<const uint4*>(crow);
#pragma unroll
      for (int i = 0; i < 8; ++i) pf[i] = src[i];
    }
  }
#pragma unroll 1
  for (int ch = 0; ch < NCH; ++ch) {
    uint32_t r[32];
    LP_TMEM_LD32(t_row + ch * 32, r);
    tc_wait_ld();
    if constexpr (ES == 2) {
      uint32_t w[16];
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        __nv_bfloat162 h = __floats2bfloat162_rn(__uint_as_float(r[2 * i]), __uint_as_float(r[2 * i + 1]));
        w[i] = *reinterpret_cast<uint32_t*>(&h);  // even column in the low half (Reading R6)
      }
      uint4* dst = reinterpret_cast<uint4*>(crow + ch * 32);
#pragma unroll
      for (int i = 0; i < 4; ++i) st_c16(dst + i, make_uint4(w[4 * i], w[4 * i + 1], w[4 * i + 2], w[4 * i + 3]));
      if constexpr (MASK != 0) {
        // byte position of word 0 of this chunk inside its region's stream
        const uint32_t pos0 = REG == 128 ? (uint32_t)(row_in_tile * 128 * ES + ((n0 + ch * 32) & 127) * ES + 1)
                                         : (uint32_t)(lane * 32 * ES + 1);
#pragma unroll
        for (int i = 0; i < 4; ++i) part.add4(w[4 * i], w[4 * i + 1], w[4 * i + 2], w[4 * i + 3], pos0 + 16 * i);
      }
    } else {
      uint4* dst = reinterpret_cast<uint4*>(crow + ch * 32);
      if (add_prev) {
        // software pipeline: this group's previous partial sums were loaded last iteration;
        // issue the next group's loads before consuming them
        uint4 prev[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) prev[i] = pf[i];
        if (ch + 1 < NCH) {
          const uint4* nxt = reinterpret_cast<const uint4*>(crow + (ch + 1) * 32);
#pragma unroll
          for (int i = 0; i < 8; ++i) pf[i] = nxt[i];
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          r[4 * i + 0] = __float_as_uint(__fadd_rn(__uint_as_float(prev[i].x), __uint_as_float(r[4 * i + 0])));
          r[4 * i + 1] = __float_as_uint(__fadd_rn(__uint_as_float(prev[i].y), __uint_as_float(r[4 * i + 1])));
          r[4 * i + 2] = __float_as_uint(__fadd_rn(__uint_as_float(prev[i].z), __uint_as_float(r[4 * i + 2])));
          r[4 * i + 3] = __float_as_uint(__fadd_rn(__uint_as_float(prev[i].w), __uint_as_float(r[4 * i + 3])));
        }
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) st_c16(dst + i, make_uint4(r[4 * i], r[4 * i + 1], r[4 * i + 2], r[4 * i + 3]));
      if (!final_pass) continue;
      if constexpr (MASK != 0) {
        const uint32_t pos0 = REG == 128 ? (uint32_t)(row_in_tile * 128 * ES + ((n0 + ch * 32) & 127) * ES + 1)
                                         : (uint32_t)(lane * 32 * ES + 1);
#pragma unroll
        for (int i = 0; i < 8; ++i) part.add4(r[4 * i], r[4 * i + 1], r[4 * i + 2], r[4 * i + 3], pos0 + 16 * i);
      }
    }
    if constexpr (MASK != 0) {
      if constexpr (REG == 32) {
        // one 32x32 region = this warp's 32 rows x this 32-column chunk
        const CkRecord rec = warp_reduce<MASK>(part);
        if (lane == 0) {
          const int64_t p = m128 * (kBM / 32) + wq, q = (n0 + ch * 32) / 32;
          const int64_t rid = p * Qr + q;
          uint32_t words[3];
          record_words<MASK>(rec, (uint64_t)32 * 32 * ES, words);
          store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
        }
        part = CkPartial<MASK>();
      } else if ((ch & 3) == 3 || ch == NCH - 1) {
        // end of a 128-column region (or of a 64-column slice of one): warp partial -> shared slot
        const CkRecord rec = warp_reduce<MASK>(part);
        if (lane == 0) srec_acc[(ch / 4) * 4 + wq] = rec;
        part = CkPartial<MASK>();
      }
    }
  }
}

// 128x128 regions: after the epilogue warps' named barrier, combine the 4 warp
// partials of each region (Listing 3's block combine) and store the record.
template <typename OutT, uint32_t MASK, int BN, int STORE>
__device__ __forceinline__ void epi_finish_128(int warp, int lane, const CkRecord* srec_acc, uint32_t* __restrict__ ck,
                                               int64_t m128, int64_t n0, int64_t Qr, int64_t rid_offset) {
  constexpr int ES = (int)sizeof(OutT);
  named_bar_epi();
  if (warp == kEpiWarp0 && lane < BN / 128) {
    const int j = lane;
    CkRecord rr = srec_acc[j * 4 + 0];
#pragma unroll
    for (int w = 1; w < 4; ++w) rr = combine(rr, srec_acc[j * 4 + w]);
    const int64_t rid = m128 * Qr + n0 / 128 + j;
    uint32_t words[3];
    record_words<MASK>(rr, (uint64_t)128 * 128 * ES, words);
    store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
  }
}

// Same for a tile stored as two 128-column halves at n_lo and (if has_hi) n_hi --
// contiguous in full runs, two column panels in paired recovery: one barrier, lane
// h of the first epilogue warp finishes half h.
template <typename OutT, uint32_t MASK, int STORE>
__device__ __forceinline__ void epi_finish_halves(int warp, int lane, const CkRecord* srec_acc,
                                                  uint32_t* __restrict__ ck, int64_t m128, int64_t n_lo, int64_t n_hi,
                                                  bool has_hi, int64_t Qr, int64_t rid_offset) {
  constexpr int ES = (int)sizeof(OutT);
  named_bar_epi();
  if (warp == kEpiWarp0 && (lane == 0 || (lane == 1 && has_hi))) {
    const int j = lane;
    CkRecord rr = srec_acc[j * 4 + 0];
#pragma unroll
    for (int w = 1; w < 4; ++w) rr = combine(rr, srec_acc[j * 4 + w]);
    const int64_t rid = m128 * Qr + (j ? n_hi : n_lo) / 128;
    uint32_t words[3];
    record_words<MASK>(rr, (uint64_t)128 * 128 * ES, words);
    store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
  }
}

// One 128x64 slice of a 128x128 region (recovery of 128x128 regions as slices): combine the 4 warp
// partials of the slice, publish them as half h of the region's partial record in the workspace, and
// let the second of the region's two slices to finish -- in this task or another CTA's -- combine both
// halves and store the record (the record words depend only on the combined sums, not on the order).
// Ordering: partial store, gpu-scope fence, arrival RMW; the finisher fences before reading the other
// half through L2 and resets the counter for the next recovery.
template <typename OutT, uint32_t MASK, int STORE>
__device__ __forceinline__ void epi_finish_slice128(int warp, int lane, const CkRecord* srec_slot,
                                                    uint32_t* __restrict__ ck, int64_t m128, int64_t n0, int64_t Qr,
                                                    int64_t rid_offset, CkRecord* part, uint32_t* cnt) {
  constexpr int ES = (int)sizeof(OutT);
  named_bar_epi();
  if (warp == kEpiWarp0 && lane == 0) {
    CkRecord rr = srec_slot[0];
#pragma unroll
    for (int w = 1; w < 4; ++w) rr = combine(rr, srec_slot[w]);
    const int64_t rid = m128 * Qr + n0 / 128;
    const int h = (int)((n0 >> 6) & 1);
    volatile uint32_t* dst = reinterpret_cast<volatile uint32_t*>(part + 2 * rid + h);
    dst[0] = rr.mod;
    dst[1] = rr.xr;
    dst[2] = rr.s;
    dst[3] = rr.wmod;
    __threadfence();
    if (atomicAdd(cnt + rid, 1u) == 1u) {
      __threadfence();
      const volatile uint32_t* o = reinterpret_cast<const volatile uint32_t*>(part + 2 * rid + (h ^ 1));
      const CkRecord other{o[0], o[1], o[2], o[3]};
      rr = combine(rr, other);
      cnt[rid] = 0u;
      uint32_t words[3];
      record_words<MASK>(rr, (uint64_t)128 * 128 * ES, words);
      store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
    }
  }
}

__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cluster address of the same variable in CTA rank 0 of the cluster
__device__ __forceinline__ uint32_t mapa_rank0(const void* p) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(smem_u32(p)));
  return r;
}
// shared::cluster address of the same variable in CTA `r` of the cluster
__device__ __forceinline__ uint32_t mapa_peer(const void* p, uint32_t r) {
  uint32_t a;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(smem_u32(p)), "r"(r));
  return a;
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void tma_load_2d_pair(const CUtensorMap* map, uint32_t mbar_rank0, void* dst, int c0,
                                                 int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, "
      "%4}], [%2];" ::"r"(smem_u32(dst)),
      "l"((uint64_t)map), "r"(mbar_rank0), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tc_mma_pair(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                            uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void tc_commit_pair(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}

}  // namespace
}  // namespace lp
