// tmm_tc.cu -- LP-protected tiled matrix multiply on the 5th-generation tensor cores.
//
// The region body of the paper's TMM (Listing 2, Listing 6)
// is a dense contraction, so on sm_100a it runs on tcgen05: operands staged in
// shared memory by TMA (cp.async.bulk.tensor, 128-B swizzle), one elected
// thread issuing tcgen05.mma (kind::f16, bf16 x bf16 -> fp32) into a TMEM
// accumulator, and 4 epilogue warps that read the accumulator back with
// tcgen05.ld.  Persistent CTAs (one per SM) walk the tile list; TMEM holds two
// 128x256 accumulators so the epilogue of tile i overlaps the mainloop of
// tile i+1 -- which is where the LP checksum work (L192) hides.
//
// LP epilogue (MASK != 0), fused in registers, no extra pass over C:
//   * every thread owns one output row of the tile (TMEM lane) and folds the
//     exact 32-bit words it stores -- bf16 pairs packed even-column-low, or
//     fp32 bits (L260-261 Fig. 2, Readings R2, R6) -- into MOD / XOR / Adler
//     partials (L192 §IV-B);
//   * 32x32 regions: one warp-wide redux.sync per checksum per region
//     (Listing 4) and lane 0 stores the record;
//   * 128x128 regions: warp redux + a 4-slot shared-memory combine across the
//     epilogue warps (Listing 3, named barrier among them only);
//   * the record goes to table[rid] with one plain store, no lock, no atomic,
//     no fence (hash-table-less global array, L349 §V), or through the hash
//     ablation (L265-274).
//
// Warp roles (192 threads): warp 0 = TMA producer, warp 1 = TMEM allocator +
// MMA issuer, warps 2..5 = epilogue (TMEM lane quarter = warp % 4).
// Region <-> tile: a 128x128 region is half of a 128x256 tile (or a whole
// 128x128 tile in list mode); a 32x32 region is one warp x 32-column chunk.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "lp_device.cuh"
#include "lp_internal.h"
#include "lp_ptx.cuh"
#include "lp_tma.h"
#include "tc_common.cuh"

namespace lp {
namespace {

constexpr int kBK = 64;      // 64 bf16 = 128 B = one swizzle atom row
constexpr int kUmmaK = 16;   // K per tcgen05.mma kind::f16
constexpr int kThreads = 192;

template <int BN>
struct TcCfg {
  static constexpr int kStages = BN == 256 ? 4 : 6;
  static constexpr int kABytes = kBM * kBK * 2;            // 16 KiB
  static constexpr int kBBytes = kBK * BN * 2;             // 32 / 16 KiB
  static constexpr int kStageBytes = kABytes + kBBytes;
  static constexpr int kTmemCols = 2 * BN;                 // two accumulators
  static constexpr int kSmemBytes = kStages * kStageBytes + 1024 /*barriers etc.*/ + 1024 /*align slack*/;
};

// Instruction descriptor kind::f16: D fp32 [4,6)=1, A bf16 [7,10)=1, B bf16 [10,13)=1,
// A K-major (bit 15 = 0), B MN-major (bit 16 = 1), N>>3 at [17,23), M>>4 at [24,29).
template <int BN>
__host__ __device__ constexpr uint32_t instr_desc() {
  return (1u << 4) | (1u << 7) | (1u << 10) | (0u << 15) | (1u << 16) | ((uint32_t)(BN >> 3) << 17) |
         ((uint32_t)(kBM >> 4) << 24);
}

__device__ __forceinline__ uint32_t instr_desc_n(int n) {
  return (1u << 4) | (1u << 7) | (1u << 10) | (0u << 15) | (1u << 16) | ((uint32_t)(n >> 3) << 17) |
         ((uint32_t)(kBM >> 4) << 24);
}

template <typename OutT, uint32_t MASK, int REG, int BN, int STORE>
__global__ void __launch_bounds__(kThreads, 1)
    tmm_tc_kernel(const __grid_constant__ CUtensorMap tmap_a, const __grid_constant__ CUtensorMap tmap_b,
                  OutT* __restrict__ C, int64_t ldc, int64_t K, TileSrc src, uint32_t* __restrict__ ck) {
  using Cfg = TcCfg<BN>;
  constexpr int S = Cfg::kStages;

  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;
  uint8_t* sB = smem + S * Cfg::kABytes;
  uint64_t* full = (uint64_t*)(smem + S * Cfg::kStageBytes);
  uint64_t* empty = full + S;
  uint64_t* tfull = empty + S;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_holder = (uint32_t*)(tempty + 2);
  CkRecord* srec = (CkRecord*)(tmem_holder + 4);  // [2 acc][BN/128 regions][4 warps]

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_a) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_b) : "memory");
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], 4);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_holder)),
                 "r"((uint32_t)Cfg::kTmemCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_holder;
  // list mode is launched programmatically dependent on the grouping kernel: the prologue above
  // (barriers, TMEM allocation, tensor-map prefetch) overlaps its tail; the task list is read only
  // after it has completed and flushed (a no-op for ordinary launches)
  asm volatile("griddepcontrol.wait;" ::: "memory");

  const int64_t ntiles = src.count();
  const int nkb = (int)(K / kBK);

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        // B is staged as 64-column chunks: 0,1 from the low half's panel, 2,3 from the high half's
        // (slice tasks: chunk c from slice c's panel)
        int64_t mb, col[4];
        int nch;
        if (BN == 256 && src.slice64) {
          src.slices(t, mb, nch, col);
        } else {
          int64_t n_lo, n_hi;
          bool has_hi;
          src.cols<BN>(t, mb, n_lo, n_hi, has_hi);
          nch = has_hi ? 4 : 2;
#pragma unroll
          for (int c = 0; c < 4; ++c) col[c] = (c < 2 ? n_lo : n_hi) + (c & 1) * 64;
        }
        const int m0 = (int)(mb * kBM);
        const uint32_t bytes = Cfg::kABytes + nch * (kBK * 128);
        // recovery reads cold operands (random failed tiles, L2 flushed): keep l2_prefetch k-blocks of this
        // task's A and B boxes in flight into L2 beyond the smem ring, so the ring's TMA loads hit L2
        const int pf = src.l2_prefetch;
        auto prefetch = [&](int kb) {
          tma_prefetch_2d(&tmap_a, kb * kBK, m0);
#pragma unroll
          for (int c = 0; c < BN / 64; ++c)
            if (c < nch) tma_prefetch_2d(&tmap_b, (int)col[c], kb * kBK);
        };
        for (int kb = 0; kb < pf && kb < nkb; ++kb) prefetch(kb);
        for (int kb = 0; kb < nkb; ++kb) {
          if (pf && kb + pf < nkb) prefetch(kb + pf);
          mbar_wait(&empty[stage], phase ^ 1);
          mbar_expect_tx(&full[stage], bytes);
          tma_load_2d(&tmap_a, &full[stage], sA + stage * Cfg::kABytes, kb * kBK, m0);
#pragma unroll
          for (int c = 0; c < BN / 64; ++c) {
            if (c >= nch) break;
            tma_load_2d(&tmap_b, &full[stage], sB + stage * Cfg::kBBytes + c * (kBK * 128), (int)col[c], kb * kBK);
          }
          if (++stage == S) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    // ===================== MMA issuer (one thread) =====================
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        // N = 256 when both halves are live, else N = 128 into the low half; slice tasks: N = 64 x slices
        uint32_t idesc;
        if (BN == 256 && src.slice64) {
          idesc = instr_desc_n(64 * ((src.tasks[t] & 3) + 1));
        } else {
          int64_t mb, n_lo, n_hi;
          bool has_hi;
          src.cols<BN>(t, mb, n_lo, n_hi, has_hi);
          idesc = (BN == 256 && has_hi) ? instr_desc<256>() : instr_desc<128>();
        }
        mbar_wait(&tempty[acc], acc_phase ^ 1);  // epilogue drained this accumulator
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + (uint32_t)(acc * BN);
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t a_addr = smem_u32(sA + stage * Cfg::kABytes);
          const uint32_t b_addr = smem_u32(sB + stage * Cfg::kBBytes);
#pragma unroll
          for (int k = 0; k < kBK / kUmmaK; ++k) {
            // A: K-major SW128, +32 B per K=16 step inside the 128-B atom; SBO = 8 rows * 128 B.
            const uint64_t ad = smem_desc(a_addr + k * kUmmaK * 2, 16, 1024);
            // B: MN-major SW128, LBO = stride between 64-column chunks, SBO = 8 K-rows * 128 B,
            //    +16 K-rows * 128 B per step.
            const uint64_t bd = smem_desc(b_addr + k * kUmmaK * 128, kBK * 128, 1024);
            tc_mma(d_tmem, ad, bd, idesc, (kb | k) ? 1u : 0u);
          }
          tc_commit(&empty[stage]);  // frees the smem slot when these MMAs complete
          if (++stage == S) {
            stage = 0;
            phase ^= 1;
          }
        }
        tc_commit(&tfull[acc]);  // accumulator ready for the epilogue
        if (++acc == 2) {
          acc = 0;
          acc_phase ^= 1;
        }
      }
    }
  } else {
    // ===================== epilogue (4 warps, 128 threads) =====================
    const int wq = warp & 3;              // TMEM lane quarter owned by this warp
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const uint32_t t_row = tmem_base + ((uint32_t)(wq * 32) << 16) + (uint32_t)(acc * BN);
      CkRecord* srec_acc = srec + acc * (BN / 128) * 4;
      if constexpr (REG == 128 && BN == 256 && MASK != 0) {
        if (src.slice64) {
          // slice task of 128x128 regions: accumulator columns [64c, 64c+64) = half of region (mb, nc[c] / 128);
          // the two warp-partial slot sets alternate so the next slice cannot overwrite a set before the
          // combining warp has read it (it passes the next slice's named barrier only after reading)
          int64_t mb, nc[4];
          int cnt;
          src.slices(t, mb, cnt, nc);
#pragma unroll 1
          for (int c = 0; c < cnt; ++c) {
            CkRecord* slot = srec_acc + (c & 1) * 4;
            epi_store<OutT, MASK, REG, 64, STORE>(t_row + 64 * c, C, ldc, mb, nc[c], wq, lane, slot, ck, src.Qr,
                                                  src.rid_offset);
            if (c == cnt - 1) {
              tc_fence_before();
              __syncwarp();
              if (lane == 0) mbar_arrive(&tempty[acc]);
            }
            epi_finish_slice128<OutT, MASK, STORE>(warp, lane, slot, ck, mb, nc[c], src.Qr, src.rid_offset, src.part,
                                                   src.cnt);
          }
          if (++acc == 2) {
            acc = 0;
            acc_phase ^= 1;
          }
          continue;
        }
      }
      if constexpr (REG == 32 && BN == 256) {
        if (src.slice64) {
          // accumulator columns [64c, 64c+64) -> slice c (32x32 records per 32-column chunk)
          int64_t mb, nc[4];
          int cnt;
          src.slices(t, mb, cnt, nc);
#pragma unroll 1
          for (int c = 0; c < cnt; ++c)
            epi_store<OutT, MASK, REG, 64, STORE>(t_row + 64 * c, C, ldc, mb, nc[c], wq, lane, srec_acc, ck, src.Qr,
                                                  src.rid_offset);
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&tempty[acc]);
          if (++acc == 2) {
            acc = 0;
            acc_phase ^= 1;
          }
          continue;
        }
      }
      int64_t mb, n_lo, n_hi;
      bool has_hi;
      src.cols<BN>(t, mb, n_lo, n_hi, has_hi);
      epi_store<OutT, MASK, REG, 128, STORE>(t_row, C, ldc, mb, n_lo, wq, lane, srec_acc, ck, src.Qr,
                                             src.rid_offset);
      if (BN == 256 && has_hi)
        epi_store<OutT, MASK, REG, 128, STORE>(t_row + 128, C, ldc, mb, n_hi, wq, lane, srec_acc + 4, ck, src.Qr,
                                               src.rid_offset);
      // all TMEM reads of this accumulator are complete (wait::ld): release it
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[acc]);
      if constexpr (MASK != 0 && REG == 128)
        epi_finish_halves<OutT, MASK, STORE>(warp, lane, srec_acc, ck, mb, n_lo, n_hi, BN == 256 && has_hi, src.Qr,
                                             src.rid_offset);
      if (++acc == 2) {
        acc = 0;
        acc_phase ^= 1;
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                 "r"((uint32_t)Cfg::kTmemCols)
                 : "memory");
  }
}

// ---------------------------------------------------------------------------- CTA-pair kernel
// Full (non-list) runs with M % 256 == 0 and N % 256 == 0 use a 2-SM CTA pair
// (cluster of 2): one tcgen05.mma.cta_group::2 computes a 256x256x16 step with
// A split by rows (128 per CTA) and B split by columns (128 per CTA), so each
// SM stages only half of B: 32 KiB per stage, a 6-deep TMA ring, and half the
// per-SM operand traffic of the 1-CTA 128x256 tile.  The leader CTA (rank 0)
// owns the smem-full barriers (both CTAs' TMA complete_tx on it) and issues the
// MMAs; commits multicast to both CTAs' barriers.  Each CTA's TMEM holds its
// 128 rows x 256 fp32 columns, double-buffered, and its 4 epilogue warps run the
// same LP epilogue as the 1-CTA kernel on its own 128 rows.
constexpr int kStages2 = 6;
constexpr int kA2Bytes = kBM * kBK * 2;   // 16 KiB: this CTA's 128 rows of A
constexpr int kB2Bytes = kBK * 128 * 2;   // 16 KiB: this CTA's 128 columns of B
constexpr int kStage2Bytes = kA2Bytes + kB2Bytes;
constexpr int kSmem2Bytes = kStages2 * kStage2Bytes + 1024 + 1024;

// ---------------------------------------------------------------------------- Listing 7 check phase
// Same-grid check-and-recover (Listing 7; NEXT row N2): before its mainloop, every CTA
// validates its 128-row half of each 256x256 tile its pair owns in the ordinary persistent
// schedule (L183: "fetching the corresponding data from memory, computing their checksums, and
// then comparing them with the ones stored in the checksum table").  Work item = one 32-row band
// (32x32 regions) or a whole 128-row half (128x128 regions) of a tile; the 6 warps take items
// round robin, lane l reads 16-byte chunk l (+32) of every row (coalesced 512-B rows), each lane's
// chunks stay inside one region column, so a segmented warp reduction yields the records.  A
// failed region sets its tile-half's bit (2 bits per tile) in this CTA's shared bitmask and bumps *d_rec;
// a tile with one failed half is recomputed as a 256x128 tile (N = 128), else as the full 256x256.
// rows of 16-B loads in flight per lane in the check phase (32 for bf16, 16 for fp32 rows of two chunks:
// 128 registers of loads; the kernel has the register file to itself at 1 CTA per SM)
#ifndef LP_CHECK_ROWS
#define LP_CHECK_ROWS 32
#endif

__device__ __forceinline__ uint4 ld_u4_noalloc(const void* p) {
  uint4 r;
  asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

template <typename OutT, uint32_t MASK, int REG, int STORE>
__device__ __forceinline__ void check_tiles(const OutT* __restrict__ C, int64_t ldc, const uint32_t* __restrict__ ck,
                                            int64_t ntiles, int64_t pair, int64_t npairs, int64_t num_m,
                                            int64_t num_n, int64_t Qr, int64_t rid_offset, uint32_t rank,
                                            uint32_t* s_fail, int64_t* d_rec) {
  constexpr int ES = (int)sizeof(OutT);
  constexpr int S = selem_of(MASK);
  constexpr int CPR = 256 * ES / 16;            // 16-byte chunks per tile-half row (32 bf16 / 64 fp32)
  constexpr int U = CPR / 32;                   // chunks per lane per row
  constexpr int CPRR = REG * ES / 16;           // chunks per region row
  constexpr int LGL = CPRR >= 32 ? 5 : (CPRR == 16 ? 4 : (CPRR == 8 ? 3 : 2));
  constexpr int RB = REG == 32 ? 32 : 128;      // rows per work item
  constexpr int NB = 128 / RB;                  // items per tile half
  constexpr int kCheckUnroll = (LP_CHECK_ROWS / U) < RB ? (LP_CHECK_ROWS / U) : RB;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t nloc = (ntiles - pair + npairs - 1) / npairs;
  for (int64_t it = warp; it < nloc * NB; it += kThreads / 32) {
    const int64_t lt = it / NB;
    const int band = (int)(it - lt * NB);
    int64_t mb, nb;
    tile_coords(pair + lt * npairs, num_m, num_n, mb, nb);
    const int64_t row0 = (mb * 2 + rank) * 128 + band * RB;
    const uint8_t* base = reinterpret_cast<const uint8_t*>(C + row0 * ldc + nb * 256);
    CkPartial<MASK> part[U];
#pragma unroll 1
    for (int r0 = 0; r0 < RB; r0 += kCheckUnroll) {
      uint4 v[kCheckUnroll][U];
#pragma unroll
      for (int r = 0; r < kCheckUnroll; ++r)
#pragma unroll
        for (int u = 0; u < U; ++u) v[r][u] = ld_u4_noalloc(base + (int64_t)(r0 + r) * ldc * ES + (lane + 32 * u) * 16);
#pragma unroll
      for (int r = 0; r < kCheckUnroll; ++r)
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int c = lane + 32 * u;
          const uint32_t pos = (uint32_t)(((r0 + r) % REG) * REG * ES + (c % CPRR) * 16 + 1);
          part[u].add4(v[r][u].x, v[r][u].y, v[r][u].z, v[r][u].w, pos);
        }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const CkRecord rec = segment_reduce<MASK>(part[u], LGL);
      const int c = lane + 32 * u;
      if ((c % CPRR) == 0) {
        const int64_t p = row0 / REG, q = nb * (256 / REG) + c / CPRR;
        const int64_t rid = p * Qr + q;
        uint32_t w[3];
        record_words<MASK>(rec, (uint64_t)REG * REG * ES, w);
        bool bad = false;
        if constexpr (STORE == 0) {
#pragma unroll
          for (int s2 = 0; s2 < S; ++s2) bad |= (ck[rid * S + s2] != w[s2]);
        } else {
          uint32_t stored[3];
          bad = !store_lookup<S, STORE>(ck, (uint32_t)(rid + rid_offset), stored);
#pragma unroll
          for (int s2 = 0; s2 < S; ++s2) bad |= (!bad && stored[s2] != w[s2]);
        }
        if (bad) {
          // two bits per tile: which 128-column half holds the failed region
          const int h = (int)((c / CPRR) * REG / 128);
          atomicOr(&s_fail[lt >> 4], 1u << (2 * (lt & 15) + h));
          atomicAdd(reinterpret_cast<unsigned long long*>(d_rec), 1ull);
        }
      }
    }
  }
}

// Tile walk of a CTA pair.  CHECK 0: the persistent schedule t = pair, pair + npairs, ...; 1 (Listing 7,
// static): the same schedule, skipping tiles whose two half bits are clear in the pair's merged bitmask
// `todo` (2 bits per local tile); 2 (Listing 7, balanced): the j-th failed tile of the GLOBAL bitmask (2 bits
// per tile id, ascending tile index) goes to pair j % npairs -- every role of both CTAs derives the same
// sequence from the bitmask, no broadcast needed.  half = which 128-column halves to compute (bit 0 / 1).
template <int CHECK>
struct TileWalk {
  int64_t t, lt, pair, npairs, ntiles;
  const uint32_t* todo;   // CHECK 1: shared bitmask over local indices
  const uint32_t* gbits;  // CHECK 2: global bitmask over tile ids
  int64_t w, nwords, j;
  uint32_t cur;
  __device__ __forceinline__ TileWalk(int64_t pair_, int64_t npairs_, int64_t ntiles_, const uint32_t* todo_,
                                      const uint32_t* gbits_)
      : t(pair_ - npairs_), lt(-1), pair(pair_), npairs(npairs_), ntiles(ntiles_), todo(todo_), gbits(gbits_), w(-1),
        nwords((ntiles_ + 15) >> 4), j(0), cur(0u) {}
  __device__ __forceinline__ bool next(int64_t& out, int& half) {
    if constexpr (CHECK == 2) {
      for (;;) {
        while (cur == 0u) {
          if (++w >= nwords) return false;
          cur = __ldcg(gbits + w);
        }
        const int b = (__ffs(cur) - 1) >> 1;  // tile slot in this word
        const uint32_t m = (cur >> (2 * b)) & 3u;
        cur &= ~(3u << (2 * b));
        const bool mine = (j % npairs) == pair;
        ++j;
        if (mine) {
          out = w * 16 + b;
          half = (int)m;
          return true;
        }
      }
    } else {
      for (;;) {
        t += npairs;
        ++lt;
        if (t >= ntiles) return false;
        half = 3;
        if (CHECK == 1) {
          half = (int)((todo[lt >> 4] >> (2 * (lt & 15))) & 3u);
          if (!half) continue;
        }
        out = t;
        return true;
      }
    }
  }
};

template <typename OutT, uint32_t MASK, int REG, int STORE, int CHECK = 0>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
    tmm_tc2_kernel(const __grid_constant__ CUtensorMap tmap_a, const __grid_constant__ CUtensorMap tmap_b,
                   OutT* __restrict__ C, int64_t ldc, int64_t K, int64_t num_m, int64_t num_n, int64_t Qr,
                   int64_t rid_offset, uint32_t* __restrict__ ck, int64_t* __restrict__ d_rec,
                   uint32_t* __restrict__ gbits, uint32_t* __restrict__ gbar) {
  constexpr int BN = 256;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;
  uint8_t* sB = smem + kStages2 * kA2Bytes;
  uint64_t* full = (uint64_t*)(smem + kStages2 * kStage2Bytes);
  uint64_t* empty = full + kStages2;
  uint64_t* tfull = empty + kStages2;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_holder = (uint32_t*)(tempty + 2);
  CkRecord* srec = (CkRecord*)(tmem_holder + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const int64_t pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmap_a);
    prefetch_tmap(&tmap_b);
    for (int s = 0; s < kStages2; ++s) {
      mbar_init(&full[s], 2);   // one arrival per CTA's producer (+ both CTAs' TMA bytes), used in rank 0
      mbar_init(&empty[s], 1);  // leader's MMA commit (multicast)
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], 8);  // 4 epilogue warps x 2 CTAs, used in rank 0
    }
    fence_barrier_init();
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_holder)),
                 "r"(512u)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_holder;
  const int64_t ntiles = num_m * num_n;
  const int nkb = (int)(K / kBK);
  // Listing 7 form: failed-tile bitmask of this pair's local tile sequence (own half | peer half)
  uint32_t* s_fail = reinterpret_cast<uint32_t*>(srec + 16);
  const int64_t nloc = (ntiles - pair + npairs - 1) / npairs;
  const int nwords = (int)((nloc + 15) >> 4);  // 2 bits per local tile
  uint32_t* s_todo = s_fail + nwords;
  if constexpr (CHECK != 0) {
    for (int i = threadIdx.x; i < nwords; i += kThreads) s_fail[i] = 0u;
    __syncthreads();
    check_tiles<OutT, MASK, REG, STORE>(C, ldc, ck, ntiles, pair, npairs, num_m, num_n, Qr, rid_offset, rank, s_fail,
                                        d_rec);
    if constexpr (CHECK == 1) {
      cluster_sync_all();  // both halves checked; the peer's bitmask is final
      uint32_t peer;
      for (int i = threadIdx.x; i < nwords; i += kThreads) {
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(peer) : "r"(mapa_peer(&s_fail[i], rank ^ 1u)) : "memory");
        s_todo[i] = s_fail[i] | peer;
      }
      __syncthreads();
    } else {
      // publish this CTA's failed tiles to the global bitmask, then a grid barrier (cooperative launch:
      // every CTA is resident); afterwards every pair reads the same global bitmask
      __syncthreads();
      for (int i = threadIdx.x; i < nwords; i += kThreads) {
        uint32_t m = s_fail[i];
        while (m) {
          const int bit = __ffs(m) - 1;
          m &= m - 1u;
          const int64_t lt = (int64_t)i * 16 + (bit >> 1);
          const int64_t t = pair + lt * npairs;
          atomicOr(gbits + (t >> 4), 1u << (2 * (t & 15) + (bit & 1)));
        }
      }
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(gbar, 1u);
        uint32_t v;
        do {
          __nanosleep(64);
          asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(gbar) : "memory");
        } while (v < gridDim.x);
      }
      __syncthreads();
    }
  }

  if (warp == 0) {
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      TileWalk<CHECK> walk(pair, npairs, ntiles, s_todo, gbits);
      int64_t t;
      int half;
      while (walk.next(t, half)) {
        int64_t mb, nb;
        tile_coords(t, num_m, num_n, mb, nb);
        // N = 256: each CTA stages 128 columns of B; one failed half (N = 128): 64 columns of that half
        const int nw = half == 3 ? 256 : 128, hoff = half == 2 ? 128 : 0;
        const int m0 = (int)(mb * 256 + rank * 128), n0 = (int)(nb * 256 + hoff + rank * (nw / 2));
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          const uint32_t full0 = mapa_rank0(&full[stage]);
          if (rank == 0)
            mbar_expect_tx(&full[stage], 2 * (kA2Bytes + (nw / 2) * kBK * 2));
          else
            mbar_arrive_remote(full0);
          tma_load_2d_pair(&tmap_a, full0, sA + stage * kA2Bytes, kb * kBK, m0);
          tma_load_2d_pair(&tmap_b, full0, sB + stage * kB2Bytes, n0, kb * kBK);
          if (nw == 256) tma_load_2d_pair(&tmap_b, full0, sB + stage * kB2Bytes + kBK * 128, n0 + 64, kb * kBK);
          if (++stage == kStages2) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      // M = 256 (cta_group::2), N = 256
      constexpr uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (0u << 15) | (1u << 16) |
                                 ((uint32_t)(256 >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      TileWalk<CHECK> walk(pair, npairs, ntiles, s_todo, gbits);
      int64_t t;
      int half;
      while (walk.next(t, half)) {
        const uint32_t idesc_t = half == 3 ? idesc : ((idesc & ~(0x3Fu << 17)) | ((uint32_t)(128 >> 3) << 17));
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + (uint32_t)(acc * BN);
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t a_addr = smem_u32(sA + stage * kA2Bytes);
          const uint32_t b_addr = smem_u32(sB + stage * kB2Bytes);
#pragma unroll
          for (int k = 0; k < kBK / kUmmaK; ++k) {
            const uint64_t ad = smem_desc(a_addr + k * kUmmaK * 2, 16, 1024);
            const uint64_t bd = smem_desc(b_addr + k * kUmmaK * 128, kBK * 128, 1024);
            tc_mma_pair(d_tmem, ad, bd, idesc_t, (kb | k) ? 1u : 0u);
          }
          tc_commit_pair(&empty[stage]);
          if (++stage == kStages2) {
            stage = 0;
            phase ^= 1;
          }
        }
        tc_commit_pair(&tfull[acc]);
        if (++acc == 2) {
          acc = 0;
          acc_phase ^= 1;
        }
      }
    }
  } else {
    const int wq = warp & 3;
    int acc = 0;
    uint32_t acc_phase = 0;
    TileWalk<CHECK> walk(pair, npairs, ntiles, s_todo, gbits);
    int64_t t;
    int half;
    while (walk.next(t, half)) {
      int64_t mb, nb;
      tile_coords(t, num_m, num_n, mb, nb);
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const uint32_t t_row = tmem_base + ((uint32_t)(wq * 32) << 16) + (uint32_t)(acc * BN);
      CkRecord* srec_acc = srec + acc * 2 * 4;
      const int64_t m128 = mb * 2 + rank;
      if (CHECK != 0 && half != 3) {
        // one failed 128-column half recomputed as 256x128: accumulator columns [0, 128) -> C columns of that half
        const int64_t n0h = nb * BN + (half == 2 ? 128 : 0);
        epi_store<OutT, MASK, REG, 128, STORE>(t_row, C, ldc, m128, n0h, wq, lane, srec_acc, ck, Qr, rid_offset);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if (rank == 0)
            mbar_arrive(&tempty[acc]);
          else
            mbar_arrive_remote(mapa_rank0(&tempty[acc]));
        }
        if constexpr (MASK != 0 && REG == 128)
          epi_finish_halves<OutT, MASK, STORE>(warp, lane, srec_acc, ck, m128, n0h, n0h, false, Qr, rid_offset);
        if (++acc == 2) {
          acc = 0;
          acc_phase ^= 1;
        }
        continue;
      }
      epi_store<OutT, MASK, REG, BN, STORE>(t_row, C, ldc, m128, nb * BN, wq, lane, srec_acc, ck, Qr, rid_offset);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if (rank == 0)
          mbar_arrive(&tempty[acc]);
        else
          mbar_arrive_remote(mapa_rank0(&tempty[acc]));
      }
      if constexpr (MASK != 0 && REG == 128)
        epi_finish_128<OutT, MASK, BN, STORE>(warp, lane, srec_acc, ck, m128, nb * BN, Qr, rid_offset);
      if (++acc == 2) {
        acc = 0;
        acc_phase ^= 1;
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  cluster_sync_all();  // the peer's remote arrivals and the leader's MMAs into both TMEMs are done
  tc_fence_after();
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(512u) : "memory");
  }
}

// ---------------------------------------------------------------------------- 256-row CTA-pair kernel
// Full runs with M % 512 == 0 and N % 256 == 0: each CTA of the pair owns a 256-row band of a 512x256
// pair tile.  Per k-step the leader issues TWO tcgen05.mma.cta_group::2 256x256x16 (pair rows = CTA rows
// [0,128) and [128,256)), into accumulators D0 / D1 that together fill the whole TMEM (512 fp32 columns).
// A is staged as one 256-row TMA box (32 KiB per k-block), B as this CTA's 128 columns (16 KiB): 48 KiB per
// 256x256x64 MACs per SM instead of 32 KiB per 128x256x64 -- 25% fewer L2 -> SM bytes per flop (the
// cuBLAS sm_100 kernel's tile shape; C5 runs power-capped, where moved bytes cost clock).  The accumulators
// cannot be double-buffered, so the epilogue drains D0 first: the next tile's D0 MMAs start while D1 drains.
constexpr int kStages4 = 4;
constexpr int kA4Bytes = 256 * kBK * 2;   // 32 KiB: this CTA's 256 rows of A
constexpr int kB4Bytes = kBK * 128 * 2;   // 16 KiB: this CTA's 128 columns of B
constexpr int kStage4Bytes = kA4Bytes + kB4Bytes;
constexpr int kSmem4Bytes = kStages4 * kStage4Bytes + 1024 + 1024;

// Work distribution of the 256-row kernel.  Static (CLC = false): persistent grid, pair p takes tiles p,
// p + npairs, ...  Cluster launch control (CLC = true): one cluster per tile in the grid; a running pair
// claims the next not-yet-launched cluster's tile with clusterlaunchcontrol.try_cancel (issued by the
// leader's producer thread, multicast to both CTAs' smem, completing 16 bytes on each CTA's clc_full
// barrier), so the tiles in flight stay a contiguous window of the raster (the order a non-persistent launch
// would run them in) while each SM keeps its TMEM / barriers / pipeline across tiles.  Every role of both
// CTAs reads each response and arrives on the leader's clc_empty for the slot (11 arrivals: 2 producers, the
// MMA thread, 8 epilogue warps) before the slot is reused.
constexpr int kClcSlots = 4;
constexpr uint32_t kClcConsumers = 11;

__device__ __forceinline__ void clc_try_cancel(uint4* resp, uint64_t* bar) {
  asm volatile(
      "clusterlaunchcontrol.try_cancel.async.shared::cta.mbarrier::complete_tx::bytes.multicast::cluster::all.b128 "
      "[%0], [%1];" ::"r"(smem_u32(resp)),
      "r"(smem_u32(bar))
      : "memory");
}
// -1: no more work (no cluster was cancelled); else the tile of the cancelled cluster (first ctaid.x / 2)
__device__ __forceinline__ int64_t clc_decode(const uint4* resp) {
  uint32_t x, valid;
  asm volatile(
      "{\n\t.reg .pred p;\n\t.reg .b128 r;\n\t"
      "ld.shared.b128 r, [%2];\n\t"
      "clusterlaunchcontrol.query_cancel.is_canceled.pred.b128 p, r;\n\t"
      "selp.u32 %1, 1, 0, p;\n\t"
      "mov.u32 %0, 0;\n\t"
      "@p clusterlaunchcontrol.query_cancel.get_first_ctaid.v4.b32.b128 {%0, _, _, _}, r;\n\t}"
      : "=r"(x), "=r"(valid)
      : "r"(smem_u32(resp))
      : "memory");
  return valid ? (int64_t)(x >> 1) : -1;
}

template <typename OutT, uint32_t MASK, int REG, int STORE, bool CLC = false>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
    tmm_tc4_kernel(const __grid_constant__ CUtensorMap tmap_a, const __grid_constant__ CUtensorMap tmap_b,
                   OutT* __restrict__ C, int64_t ldc, int64_t K, int64_t num_m, int64_t num_n, int64_t group,
                   int64_t Qr, int64_t rid_offset, uint32_t* __restrict__ ck) {
  constexpr int BN = 256;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;
  uint8_t* sB = smem + kStages4 * kA4Bytes;
  uint64_t* full = (uint64_t*)(smem + kStages4 * kStage4Bytes);
  uint64_t* empty = full + kStages4;
  uint64_t* tfull = empty + kStages4;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_holder = (uint32_t*)(tempty + 2);
  CkRecord* srec = (CkRecord*)(tmem_holder + 4);
  uint4* clc_resp = (uint4*)(srec + 16);
  uint64_t* clc_full = (uint64_t*)(clc_resp + kClcSlots);
  uint64_t* clc_empty = clc_full + kClcSlots;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const int64_t pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmap_a);
    prefetch_tmap(&tmap_b);
    for (int s = 0; s < kStages4; ++s) {
      mbar_init(&full[s], 2);
      mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], 8);  // 4 epilogue warps x 2 CTAs, used in rank 0
    }
    if constexpr (CLC) {
      for (int s = 0; s < kClcSlots; ++s) {
        mbar_init(&clc_full[s], 1);                 // this CTA's producer: arrive.expect_tx(16)
        mbar_init(&clc_empty[s], kClcConsumers);    // used in rank 0
      }
    }
    fence_barrier_init();
  }
  // next tile of this role: the static stride, or the next CLC response (fetch index i)
  int clc_i = 0;
  // whole_warp: every lane reads the response; the warp converges BEFORE lane 0 releases the slot -- a lane
  // still to read it would otherwise see the next response the leader may issue into the slot at once
  auto clc_next = [&](bool expect_tx, bool arrive, bool whole_warp = false) -> int64_t {
    const int slot = clc_i % kClcSlots;
    const uint32_t par = (uint32_t)((clc_i / kClcSlots) & 1);
    if (expect_tx) mbar_expect_tx(&clc_full[slot], 16);
    mbar_wait(&clc_full[slot], par);
    const int64_t t = clc_decode(&clc_resp[slot]);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (whole_warp) __syncwarp();
    if (arrive) {
      if (rank == 0)
        mbar_arrive(&clc_empty[slot]);
      else
        mbar_arrive_remote(mapa_rank0(&clc_empty[slot]));
    }
    ++clc_i;
    return t;
  };
  // leader producer: claim the work for fetch j (slot j % S free once fetch j - S is consumed everywhere)
  auto clc_issue = [&](int j) {
    const int slot = j % kClcSlots;
    mbar_wait(&clc_empty[slot], (uint32_t)(((j / kClcSlots) & 1) ^ 1));
    clc_try_cancel(&clc_resp[slot], &clc_full[slot]);
  };
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_holder)),
                 "r"(512u)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_holder;
  const int64_t ntiles = num_m * num_n;
  const int nkb = (int)(K / kBK);

  if (warp == 0) {
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      if (CLC && rank == 0) clc_issue(0);
      for (int64_t t = pair; CLC ? t >= 0 : t < ntiles;) {
        int64_t mb, nb;
        tile_coords_g(t, num_m, num_n, group, mb, nb);
        const int m0 = (int)(mb * 512 + rank * 256), n0 = (int)(nb * 256 + rank * 128);
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          const uint32_t full0 = mapa_rank0(&full[stage]);
          if (rank == 0)
            mbar_expect_tx(&full[stage], 2 * kStage4Bytes);
          else
            mbar_arrive_remote(full0);
          tma_load_2d_pair(&tmap_a, full0, sA + stage * kA4Bytes, kb * kBK, m0);
          tma_load_2d_pair(&tmap_b, full0, sB + stage * kB4Bytes, n0, kb * kBK);
          tma_load_2d_pair(&tmap_b, full0, sB + stage * kB4Bytes + kBK * 128, n0 + 64, kb * kBK);
          if (++stage == kStages4) {
            stage = 0;
            phase ^= 1;
          }
        }
        if constexpr (CLC) {
          t = clc_next(true, true);
          if (rank == 0 && t >= 0) clc_issue(clc_i);
        } else {
          t += npairs;
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      constexpr uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (0u << 15) | (1u << 16) |
                                 ((uint32_t)(256 >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
      int stage = 0;
      uint32_t phase = 0;
      uint32_t acc_phase = 0;
      for (int64_t t = pair; CLC ? t >= 0 : t < ntiles; t = CLC ? clc_next(false, true) : t + npairs) {
        mbar_wait(&tempty[0], acc_phase ^ 1);  // D0 drained by the previous tile's epilogue
        tc_fence_after();
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t a_addr = smem_u32(sA + stage * kA4Bytes);
          const uint32_t b_addr = smem_u32(sB + stage * kB4Bytes);
#pragma unroll
          for (int k = 0; k < kBK / kUmmaK; ++k) {
            const uint64_t bd = smem_desc(b_addr + k * kUmmaK * 128, kBK * 128, 1024);
            tc_mma_pair(tmem_base, smem_desc(a_addr + k * kUmmaK * 2, 16, 1024), bd, idesc, (kb | k) ? 1u : 0u);
            if (kb == 0 && k == 0) {
              mbar_wait(&tempty[1], acc_phase ^ 1);  // D1 drained (overlaps the D0 MMAs above)
              tc_fence_after();
            }
            tc_mma_pair(tmem_base + 256u, smem_desc(a_addr + 128 * 128 + k * kUmmaK * 2, 16, 1024), bd, idesc,
                        (kb | k) ? 1u : 0u);
          }
          tc_commit_pair(&empty[stage]);
          if (++stage == kStages4) {
            stage = 0;
            phase ^= 1;
          }
        }
        tc_commit_pair(&tfull[0]);
        tc_commit_pair(&tfull[1]);
        acc_phase ^= 1;
      }
    }
  } else if (warp >= kEpiWarp0) {
    const int wq = warp & 3;
    uint32_t acc_phase = 0;
    for (int64_t t = pair; CLC ? t >= 0 : t < ntiles;) {
      int64_t mb, nb;
      tile_coords_g(t, num_m, num_n, group, mb, nb);
#pragma unroll 1
      for (int d = 0; d < 2; ++d) {
        mbar_wait(&tfull[d], acc_phase);
        tc_fence_after();
        const uint32_t t_row = tmem_base + ((uint32_t)(wq * 32) << 16) + (uint32_t)(d * BN);
        CkRecord* srec_d = srec + d * 2 * 4;
        const int64_t m128 = mb * 4 + rank * 2 + d;
        epi_store<OutT, MASK, REG, BN, STORE>(t_row, C, ldc, m128, nb * BN, wq, lane, srec_d, ck, Qr, rid_offset);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if (rank == 0)
            mbar_arrive(&tempty[d]);
          else
            mbar_arrive_remote(mapa_rank0(&tempty[d]));
        }
        if constexpr (MASK != 0 && REG == 128)
          epi_finish_128<OutT, MASK, BN, STORE>(warp, lane, srec_d, ck, m128, nb * BN, Qr, rid_offset);
      }
      acc_phase ^= 1;
      if constexpr (CLC) {
        // every lane reads the response; lane 0 arrives for the warp once all have read it
        t = clc_next(false, lane == 0, true);
      } else {
        t += npairs;
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  cluster_sync_all();
  tc_fence_after();
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(512u) : "memory");
  }
}

// ---------------------------------------------------------------------------- host side
bool make_map_2d(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer, uint64_t ld_elems,
                 uint32_t box_inner, uint32_t box_outer) {
  return tma_map_2d(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, base, inner, outer, ld_elems, box_inner, box_outer,
                    CU_TENSOR_MAP_SWIZZLE_128B);
}

// List-mode (recovery) launches carry the programmatic-stream-serialization attribute so the CTAs
// can be scheduled while the grouping kernel (which triggers launch_dependents) is still running.
template <typename Kern, typename... Args>
cudaError_t launch_maybe_pdl(Kern kfn, unsigned grid, int smem, cudaStream_t st, bool pdl, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kfn, args...);
}

// k-blocks of L2 prefetch distance in list mode (LP_TC_PREFETCH=<n> for A/B runs; default 0 = off: measured
// slower at 4/8/16 k-blocks -- the re-execution is bound by the L2 -> SM fabric, not by DRAM latency)
int l2_prefetch_kblocks() {
  static int v = [] {
    const char* e = getenv("LP_TC_PREFETCH");
    return e ? atoi(e) : 0;
  }();
  return v;
}

template <typename OutT, int REG, int BN>
cudaError_t launch_cfg(const TmmArgs& a, cudaStream_t st, const char** why) {
  using Cfg = TcCfg<BN>;
  CUtensorMap ma, mb;
  if (!make_map_2d(&ma, a.A, (uint64_t)a.K, (uint64_t)a.M, (uint64_t)a.lda, kBK, kBM) ||
      !make_map_2d(&mb, a.B, (uint64_t)a.N, (uint64_t)a.K, (uint64_t)a.ldb, 64, kBK)) {
    *why = "cuTensorMapEncodeTiled failed";
    return cudaErrorInvalidValue;
  }
  TileSrc src;
  src.num_m = a.M / kBM;
  src.num_n = a.N / BN;
  src.list = a.list;
  src.d_n = a.d_n;
  src.rid_offset = a.rid_offset;
  src.Qr = a.N / REG;
  src.reg = REG;
  src.list_is_tiles = a.list_is_tiles;
  src.tasks = a.list ? a.tasks : nullptr;
  src.d_ntasks = a.d_ntasks;
  src.n128 = a.N / 128;
  src.slice64 = a.slice64;
  src.n64 = a.N / 64;
  src.part = reinterpret_cast<CkRecord*>(a.slice_part);
  src.l2_prefetch = a.list ? l2_prefetch_kblocks() : 0;
  src.cnt = a.slice_cnt;
  const int64_t R = (a.M / REG) * (a.N / REG);
  int64_t grid = a.list ? (R < a.sm_count ? R : a.sm_count) : src.num_m * src.num_n;
  if (grid > a.sm_count) grid = a.sm_count;
  if (grid < 1) grid = 1;
  const int smem = Cfg::kSmemBytes;
  cudaError_t e = cudaSuccess;
  const int sk = a.mask ? a.hash.store : 0;
  switch (a.mask * 5 + sk) {
#define LP_TC_CASE(M, S)                                                                                    \
  case M * 5 + S: {                                                                                         \
    auto kfn = tmm_tc_kernel<OutT, M, REG, BN, S>;                                                         \
    e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);                       \
    if (e != cudaSuccess) return e;                                                                         \
    e = launch_maybe_pdl(kfn, (unsigned)grid, smem, st, a.list != nullptr, ma, mb, (OutT*)a.C, a.ldc, a.K, src, \
                         a.ck);                                                                             \
    if (e != cudaSuccess) return e;                                                                         \
    break;                                                                                                  \
  }
#define LP_TC_CASE3(M) LP_TC_CASE(M, 0)
#define LP_TC_CASE5(M) LP_TC_CASE(M, 0) LP_TC_CASE(M, 1) LP_TC_CASE(M, 2) LP_TC_CASE(M, 3) LP_TC_CASE(M, 4)
    LP_TC_CASE(0, 0)
    LP_TC_CASE5(1)
    LP_TC_CASE3(2)
    LP_TC_CASE5(3)
    LP_TC_CASE3(4)
    LP_TC_CASE3(5)
    LP_TC_CASE3(6)
    LP_TC_CASE3(7)
#undef LP_TC_CASE3
#undef LP_TC_CASE5
#undef LP_TC_CASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

template <typename OutT, int REG>
cudaError_t launch_pair(const TmmArgs& a, cudaStream_t st, const char** why) {
  CUtensorMap ma, mb;
  if (!make_map_2d(&ma, a.A, (uint64_t)a.K, (uint64_t)a.M, (uint64_t)a.lda, kBK, kBM) ||
      !make_map_2d(&mb, a.B, (uint64_t)a.N, (uint64_t)a.K, (uint64_t)a.ldb, 64, kBK)) {
    *why = "cuTensorMapEncodeTiled failed";
    return cudaErrorInvalidValue;
  }
  const int64_t num_m = a.M / 256, num_n = a.N / 256;
  int64_t grid = 2 * num_m * num_n;
  const int64_t cap = a.sm_count & ~1;
  if (grid > cap) grid = cap;
  if (grid < 2) grid = 2;
  const int64_t Qr = a.N / REG;
  const int sk = a.mask ? a.hash.store : 0;
  cudaError_t e = cudaSuccess;
  switch (a.mask * 5 + sk) {
#define LP_TC2_CASE(M, S)                                                                                   \
  case M * 5 + S: {                                                                                         \
    auto kfn = tmm_tc2_kernel<OutT, M, REG, S>;                                                            \
    e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem2Bytes);                \
    if (e != cudaSuccess) return e;                                                                         \
    kfn<<<(unsigned)grid, kThreads, kSmem2Bytes, st>>>(ma, mb, (OutT*)a.C, a.ldc, a.K, num_m, num_n, Qr,    \
                                                       a.rid_offset, a.ck, nullptr, nullptr, nullptr);     \
    break;                                                                                                  \
  }
#define LP_TC2_CASE3(M) LP_TC2_CASE(M, 0)
#define LP_TC2_CASE5(M) LP_TC2_CASE(M, 0) LP_TC2_CASE(M, 1) LP_TC2_CASE(M, 2) LP_TC2_CASE(M, 3) LP_TC2_CASE(M, 4)
    LP_TC2_CASE(0, 0)
    LP_TC2_CASE5(1)
    LP_TC2_CASE3(2)
    LP_TC2_CASE5(3)
    LP_TC2_CASE3(4)
    LP_TC2_CASE3(5)
    LP_TC2_CASE3(6)
    LP_TC2_CASE3(7)
#undef LP_TC2_CASE3
#undef LP_TC2_CASE5
#undef LP_TC2_CASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

// LP_TC_TILE=128 forces the 128-row-per-CTA pair kernel for shapes the 256-row one takes (A/B runs);
// LP_TC4_GROUP=<n> sets its raster group (M-blocks of 512 rows per group)
int tc4_mode() {
  static int v = [] {
    const char* e = getenv("LP_TC_TILE");
    return (e && atoi(e) == 128) ? 0 : 1;
  }();
  return v;
}
// The 256-row kernel takes its tiles through cluster launch control (LP_TC_CLC=0: static persistent
// schedule, A/B): at 32768^3 DRAM reads 158 -> 98 GB, C5 65536^3 485 -> 442 ms = cuBLAS (profiles/r02/ab_clc.txt)
bool tc4_clc() {
  static bool v = [] {
    const char* e = getenv("LP_TC_CLC");
    return !(e && atoi(e) == 0);
  }();
  return v;
}
int64_t tc4_group() {
  static int64_t v = [] {
    const char* e = getenv("LP_TC4_GROUP");
    return e ? (int64_t)atoi(e) : (int64_t)0;  // 0: per launch, 4 with CLC, 2 static
  }();
  return v < 0 ? 0 : v;
}

template <typename OutT, int REG>
cudaError_t launch_pair4(const TmmArgs& a, cudaStream_t st, const char** why) {
  CUtensorMap ma, mb;
  if (!make_map_2d(&ma, a.A, (uint64_t)a.K, (uint64_t)a.M, (uint64_t)a.lda, kBK, 256) ||
      !make_map_2d(&mb, a.B, (uint64_t)a.N, (uint64_t)a.K, (uint64_t)a.ldb, 64, kBK)) {
    *why = "cuTensorMapEncodeTiled failed";
    return cudaErrorInvalidValue;
  }
  const int64_t num_m = a.M / 512, num_n = a.N / 256;
  const bool clc = tc4_clc();
  int64_t grid = 2 * num_m * num_n;  // CLC: one cluster per tile
  const int64_t cap = a.sm_count & ~1;
  if (!clc && grid > cap) grid = cap;
  if (grid < 2) grid = 2;
  if (grid > (int64_t)0x7FFFFFFF) {
    *why = "grid too large";
    return cudaErrorInvalidValue;
  }
  const int64_t Qr = a.N / REG;
  const int sk = a.mask ? a.hash.store : 0;
  const int64_t G = tc4_group() ? tc4_group() : (clc ? 4 : 2);
  cudaError_t e = cudaSuccess;
  switch (a.mask * 5 + sk) {
#define LP_TC4_CASE(M, S)                                                                                   \
  case M * 5 + S: {                                                                                         \
    auto kfn = clc ? tmm_tc4_kernel<OutT, M, REG, S, true> : tmm_tc4_kernel<OutT, M, REG, S, false>;        \
    e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmem4Bytes);                \
    if (e != cudaSuccess) return e;                                                                         \
    kfn<<<(unsigned)grid, kThreads, kSmem4Bytes, st>>>(ma, mb, (OutT*)a.C, a.ldc, a.K, num_m, num_n, G, Qr, \
                                                       a.rid_offset, a.ck);                                 \
    break;                                                                                                  \
  }
#define LP_TC4_CASE3(M) LP_TC4_CASE(M, 0)
#define LP_TC4_CASE5(M) LP_TC4_CASE(M, 0) LP_TC4_CASE(M, 1) LP_TC4_CASE(M, 2) LP_TC4_CASE(M, 3) LP_TC4_CASE(M, 4)
    LP_TC4_CASE(0, 0)
    LP_TC4_CASE5(1)
    LP_TC4_CASE3(2)
    LP_TC4_CASE5(3)
    LP_TC4_CASE3(4)
    LP_TC4_CASE3(5)
    LP_TC4_CASE3(6)
    LP_TC4_CASE3(7)
#undef LP_TC4_CASE3
#undef LP_TC4_CASE5
#undef LP_TC4_CASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

template <typename Kern, typename... Args>
cudaError_t launch_cooperative(Kern kfn, unsigned grid, int smem, cudaStream_t st, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kfn, args...);
}

template <typename OutT, int REG>
cudaError_t launch_pair_check(const TmmArgs& a, int64_t* d_rec, uint32_t* gbits, uint32_t* gbar, cudaStream_t st,
                              const char** why) {
  CUtensorMap ma, mb;
  if (!make_map_2d(&ma, a.A, (uint64_t)a.K, (uint64_t)a.M, (uint64_t)a.lda, kBK, kBM) ||
      !make_map_2d(&mb, a.B, (uint64_t)a.N, (uint64_t)a.K, (uint64_t)a.ldb, 64, kBK)) {
    *why = "cuTensorMapEncodeTiled failed";
    return cudaErrorInvalidValue;
  }
  const int64_t num_m = a.M / 256, num_n = a.N / 256;
  int64_t grid = 2 * num_m * num_n;
  const int64_t cap = a.sm_count & ~1;
  if (grid > cap) grid = cap;
  if (grid < 2) grid = 2;
  const int64_t Qr = a.N / REG;
  cudaError_t e = cudaMemsetAsync(d_rec, 0, sizeof(int64_t), st);
  if (e != cudaSuccess) return e;
  const bool balanced = gbits != nullptr && gbar != nullptr;
  if (balanced) {  // global failed-tile bitmask + grid barrier counter, cleared in stream order (one memset when
                   // the counter directly follows the bitmask, as in liblp's workspace layout)
    const size_t bits_bytes = (size_t)((num_m * num_n + 15) / 16) * 4;
    if (gbar > gbits && (size_t)((uint8_t*)gbar - (uint8_t*)gbits) <= bits_bytes + 4096) {
      e = cudaMemsetAsync(gbits, 0, (size_t)((uint8_t*)gbar - (uint8_t*)gbits) + sizeof(uint32_t), st);
    } else {
      e = cudaMemsetAsync(gbar, 0, sizeof(uint32_t), st);
      if (e == cudaSuccess) e = cudaMemsetAsync(gbits, 0, bits_bytes, st);
    }
    if (e != cudaSuccess) return e;
  }
  auto smem_for = [&](int64_t g) { return kSmem2Bytes + (int)(2 * (((num_m * num_n + g / 2 - 1) / (g / 2)) + 15) / 16 * 4); };
  switch (a.mask * 5 + a.hash.store) {
#define LP_TC2C_CASE(M, S)                                                                                  \
  case M * 5 + S: {                                                                                         \
    if (balanced) {                                                                                         \
      auto kfn = tmm_tc2_kernel<OutT, M, REG, S, 2>;                                                       \
      /* every CTA must be resident for the grid barrier: at most the co-resident clusters */              \
      int ncl = 0;                                                                                          \
      e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_for(2));             \
      if (e != cudaSuccess) return e;                                                                       \
      cudaLaunchConfig_t oc = {};                                                                           \
      oc.gridDim = dim3((unsigned)grid);                                                                    \
      oc.blockDim = dim3(kThreads);                                                                         \
      oc.dynamicSmemBytes = (size_t)smem_for(2);                                                            \
      e = cudaOccupancyMaxActiveClusters(&ncl, kfn, &oc);                                                   \
      if (e != cudaSuccess) return e;                                                                       \
      const int64_t g2 = (2 * (int64_t)ncl < grid) ? 2 * (int64_t)ncl : grid;                               \
      if (g2 < 2) { *why = "no co-resident CTA pair"; return cudaErrorInvalidValue; }                      \
      const int sm2 = smem_for(g2);                                                                         \
      if (sm2 > 227 * 1024) { *why = "too many tiles per CTA pair for the bitmask"; return cudaErrorInvalidValue; } \
      e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, sm2);                      \
      if (e != cudaSuccess) return e;                                                                       \
      e = launch_cooperative(kfn, (unsigned)g2, sm2, st, ma, mb, (OutT*)a.C, a.ldc, a.K, num_m, num_n, Qr,  \
                             a.rid_offset, a.ck, d_rec, gbits, gbar);                                       \
    } else {                                                                                                \
      const int sm1 = smem_for(grid);                                                                       \
      if (sm1 > 227 * 1024) { *why = "too many tiles per CTA pair for the bitmask"; return cudaErrorInvalidValue; } \
      auto kfn = tmm_tc2_kernel<OutT, M, REG, S, 1>;                                                       \
      e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, sm1);                      \
      if (e != cudaSuccess) return e;                                                                       \
      kfn<<<(unsigned)grid, kThreads, sm1, st>>>(ma, mb, (OutT*)a.C, a.ldc, a.K, num_m, num_n, Qr,          \
                                                 a.rid_offset, a.ck, d_rec, nullptr, nullptr);              \
    }                                                                                                       \
    if (e != cudaSuccess) return e;                                                                         \
    break;                                                                                                  \
  }
#define LP_TC2C_CASE3(M) LP_TC2C_CASE(M, 0)
#define LP_TC2C_CASE5(M) LP_TC2C_CASE(M, 0) LP_TC2C_CASE(M, 1) LP_TC2C_CASE(M, 2) LP_TC2C_CASE(M, 3) LP_TC2C_CASE(M, 4)
    LP_TC2C_CASE5(1)
    LP_TC2C_CASE3(2)
    LP_TC2C_CASE5(3)
    LP_TC2C_CASE3(4)
    LP_TC2C_CASE3(5)
    LP_TC2C_CASE3(6)
    LP_TC2C_CASE3(7)
#undef LP_TC2C_CASE3
#undef LP_TC2C_CASE5
#undef LP_TC2C_CASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

template <typename OutT, int REG>
cudaError_t launch_reg(const TmmArgs& a, cudaStream_t st, const char** why) {
  if (!a.list && a.M % 512 == 0 && a.N % 256 == 0 && !a.force_1cta && tc4_mode())
    return launch_pair4<OutT, REG>(a, st, why);
  if (!a.list && a.M % 256 == 0 && a.N % 256 == 0 && !a.force_1cta) return launch_pair<OutT, REG>(a, st, why);
  // list mode re-executes 128x128 tiles (BN = 128): one 128x128 region, or the
  // 16 32x32 regions of a de-duplicated tile; paired tasks (two such tiles of one
  // row band) run on the BN = 256 kernel with B gathered from two column panels, and
  // so do slice tasks (1-4 de-duplicated 128x64 slices of one row band, N = 64..256)
  const bool bn256 = a.list ? (a.tasks != nullptr) : (a.N % 256 == 0);
  return bn256 ? launch_cfg<OutT, REG, 256>(a, st, why) : launch_cfg<OutT, REG, 128>(a, st, why);
}

}  // namespace

bool tmm_tc_supported(int64_t M, int64_t N, int64_t K, int RM, int RN, int in_bf16, int64_t lda, int64_t ldb,
                      int64_t ldc, const void* A, const void* B, const void* C) {
  if (!in_bf16) return false;
  if (!((RM == 128 && RN == 128) || (RM == 32 && RN == 32))) return false;
  if (M % kBM || N % 128 || K % kBK || K <= 0) return false;
  if ((lda * 2) % 16 || (ldb * 2) % 16 || (ldc * 2) % 16) return false;
  if ((((uintptr_t)A) & 15u) || (((uintptr_t)B) & 15u) || (((uintptr_t)C) & 15u)) return false;
  if (M > (int64_t)INT32_MAX || N > (int64_t)INT32_MAX || K > (int64_t)INT32_MAX) return false;
  return true;
}

bool tmm_tc_check_supported(int64_t M, int64_t N) { return M % 256 == 0 && N % 256 == 0; }

cudaError_t launch_tmm_tc_check_recover(const TmmArgs& a, int64_t* d_rec, uint32_t* gbits, uint32_t* gbar,
                                        cudaStream_t st, const char** why) {
  if (a.mask == 0 || a.list || !tmm_tc_check_supported(a.M, a.N)) return cudaErrorInvalidValue;
  if (a.RM == 128)
    return a.out_bf16 ? launch_pair_check<__nv_bfloat16, 128>(a, d_rec, gbits, gbar, st, why)
                      : launch_pair_check<float, 128>(a, d_rec, gbits, gbar, st, why);
  return a.out_bf16 ? launch_pair_check<__nv_bfloat16, 32>(a, d_rec, gbits, gbar, st, why)
                    : launch_pair_check<float, 32>(a, d_rec, gbits, gbar, st, why);
}

cudaError_t launch_tmm_tc(const TmmArgs& a, cudaStream_t st, const char** why) {
  if (a.RM == 128) {
    return a.out_bf16 ? launch_reg<__nv_bfloat16, 128>(a, st, why) : launch_reg<float, 128>(a, st, why);
  }
  return a.out_bf16 ? launch_reg<__nv_bfloat16, 32>(a, st, why) : launch_reg<float, 32>(a, st, why);
}

}  // namespace lp
