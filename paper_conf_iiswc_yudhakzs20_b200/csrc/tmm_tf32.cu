// tmm_tf32.cu -- fp32 LP-protected TMM on the tensor cores via 3xTF32 (CTA pair).
//
// Listing 6's TMM is fp32 (L546-554).  An fp32 GEMM is a dense contraction, so
// on sm_100a it belongs on tcgen05 -- but kind::tf32 keeps only 10 mantissa
// bits, far from the 1e-5 fp32 tolerance (Reading R16).  Each operand is split
// exactly into x = hi + lo with hi = x with the low 13 mantissa bits cleared (a
// tf32 number) and lo = x - hi (exact in fp32), and every K step issues
//     D += Ahi*Bhi + Ahi*Blo + Alo*Bhi          (Alo*Blo, ~2^-22 relative, dropped)
// so the product error is ~2^-21 relative while the tensor pipe does the work.
// Integer-valued inputs have lo = 0 and stay exact (bit-exact tests).
//
// Structure (cluster of 2 CTAs, M = 256 x N = 256 tiles, K step 32):
//   warp 0   TMA producer: raw fp32 A rows (K-major) / B columns (row-major B,
//            i.e. MN-major) of this CTA -> a 3-deep raw ring
//   warps 6-9 converters: raw stage -> converted stage [A_hi|A_lo|B_hi|B_lo]:
//            hi = x & 0xFFFFE000, lo = x - hi; A keeps its K-major SW128 layout
//            (element-wise), B is transposed to K-major SW128 on the way (the
//            tf32 MMA reads an MN-major B operand as zeros on sm_100a --
//            measured), fence.proxy.async, then arrive on the leader's barrier
//   warp 1   (leader) MMA issuer: 3 x tcgen05.mma.cta_group::2.kind::tf32 per
//            8-wide K step from a 2-deep converted ring, commits multicast
//   warps 2-5 epilogue: per K chunk SUM += ACC in TMEM (tcgen05.ld / fadd / tcgen05.st),
//            then on the last chunk the LP epilogue of the bf16 kernels from SUM (fp32 words).
// Recovery re-runs this same kernel on a de-duplicated list of 256x256 tiles, so
// the recomputed bits equal the golden ones (same instruction sequence).
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "lp_device.cuh"
#include "lp_internal.h"
#include "lp_ptx.cuh"
#include "lp_tma.h"
#include "tc_common.cuh"

namespace lp {
namespace {

constexpr int kFBK = 32;                          // 32 fp32 = 128 B = one swizzle-atom row
constexpr int kFUmmaK = 8;                        // K per tcgen05.mma kind::tf32
#ifndef LP_TF32_RAW_HI  // the MMA reads A's hi part straight from the raw TMA stage (see below)
#define LP_TF32_RAW_HI 1
#endif
// kind::tf32 ignores the low 13 mantissa bits of its 32-bit operands (measured: raw fp32 words as the hi operand
// give bit-identical products to x & 0xFFFFE000 -- tools/probe/tf32_raw_hi.sh), so with LP_TF32_RAW_HI the
// converters write only A_lo, B_hi, B_lo and the MMA takes A_hi from the raw ring, which it then releases too.
constexpr int kFRawStages = LP_TF32_RAW_HI ? 4 : 3;   // TMA ring
constexpr int kFCvStages = 2;                     // converted ring
#ifndef LP_TF32_CONV_WARPS
#define LP_TF32_CONV_WARPS 8
#endif
#ifndef LP_TF32_BLOOP
#define LP_TF32_BLOOP 0
#endif
#ifndef LP_TF32_RAW_HI_PROBE  // probe build: does kind::tf32 ignore the low 13 mantissa bits of its operands?
#define LP_TF32_RAW_HI_PROBE 0
#endif
constexpr int kFConvWarps = LP_TF32_CONV_WARPS;   // converter warps per CTA (4: one column of B per thread)
constexpr int kFConvThreads = kFConvWarps * 32;
constexpr int kFConvWarp0 = 6;
constexpr int kFThreads = (kFConvWarp0 + kFConvWarps) * 32;  // TMA, MMA, 4 epilogue, converter warps
constexpr int kFTile = 16384;                     // one 128 x 32 fp32 operand tile
constexpr int kFRawBytes = 2 * kFTile;            // raw stage: [A (K-major)][B (MN-major, 4 x 32-col chunks)]
// converted stage: [A_hi][A_lo][B_hi][B_lo] (or [A_lo][B_hi][B_lo] with LP_TF32_RAW_HI), all K-major SW128
constexpr int kFCvBytes = (LP_TF32_RAW_HI ? 3 : 4) * kFTile;
constexpr int kFCvALo = LP_TF32_RAW_HI ? 0 : kFTile, kFCvBHi = kFCvALo + kFTile, kFCvBLo = kFCvBHi + kFTile;
constexpr int kFSmemBytes = kFRawStages * kFRawBytes + kFCvStages * kFCvBytes + 512 + 1024;
// K is accumulated in chunks of kFChunkKB x 32 = 512 in one TMEM accumulator (columns
// 0..255); after each chunk the epilogue warps fold it into a TMEM-resident running
// sum (columns 256..511) with IEEE fp32 adds and release the accumulator; C and the
// LP record are stored from the running sum after the last chunk.  The tcgen05
// fp32 accumulator is markedly less accurate than round-to-nearest (measured: error
// std 2.0e-4 vs 8.6e-6 for exact products at K = 4096, growing ~K^1.5), so long K
// runs are cut into short, freshly-zeroed chunks.  Measured at 8192^3 (normwise
// rel. error / time): chunk 512: 3.9e-6 / 5.7 ms; 1024: 7.7e-6 / 4.9 ms; 2048:
// 1.4e-5 / 4.6 ms; none: 5.9e-5 / 4.1 ms -- 512 keeps a 2.5x margin to 1e-5.
constexpr int kFChunkKB = 16;

__device__ __forceinline__ void tc_mma_pair_tf32(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                                 uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

struct PairTiles {
  int64_t num_m, num_n;   // 256x256 tile grid
  const int64_t* list;    // recovery: failed rids (or tile ids when list_is_tiles)
  const int64_t* d_n;
  int list_is_tiles;
  int64_t Qr, rid_offset;
  int reg;
  __device__ __forceinline__ int64_t count() const { return list ? *d_n : num_m * num_n; }
  __device__ __forceinline__ void coords(int64_t t, int64_t& mb, int64_t& nb) const {
    if (!list) {
      tile_coords(t, num_m, num_n, mb, nb);
    } else if (list_is_tiles) {
      mb = list[t] / num_n;
      nb = list[t] - mb * num_n;
    } else {
      const int64_t rid = list[t] - rid_offset;
      const int64_t p = rid / Qr, q = rid - p * Qr;
      mb = p * reg / 256;
      nb = q * reg / 256;
    }
  }
};

template <uint32_t MASK, int REG, int STORE>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kFThreads, 1)
    tmm_tf32x3_kernel(const __grid_constant__ CUtensorMap tmap_a, const __grid_constant__ CUtensorMap tmap_b,
                      float* __restrict__ C, int64_t ldc, int64_t K, PairTiles tiles, uint32_t* __restrict__ ck,
                      int chunk_kb) {
  constexpr int BN = 256;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* cv_base = smem + kFRawStages * kFRawBytes;
  uint64_t* raw_full = (uint64_t*)(cv_base + kFCvStages * kFCvBytes);
  uint64_t* raw_empty = raw_full + kFRawStages;
  uint64_t* cv_full = raw_empty + kFRawStages;
  uint64_t* cv_empty = cv_full + kFCvStages;
  uint64_t* tfull = cv_empty + kFCvStages;
  uint64_t* tempty = tfull + 2;
  CkRecord* srec = (CkRecord*)(tempty + 2);                       // [2 acc][2 regions][4 warps] = 256 B
  uint32_t* tmem_holder = (uint32_t*)((uint8_t*)(tempty + 2) + 256);  // own 128-B line, written by tcgen05.alloc
  auto raw = [&](int s) { return smem + s * kFRawBytes; };
  auto cvs = [&](int s) { return cv_base + s * kFCvBytes; };

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const int64_t pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmap_a);
    prefetch_tmap(&tmap_b);
    for (int s = 0; s < kFRawStages; ++s) {
      mbar_init(&raw_full[s], 1);   // this CTA's TMA bytes
      mbar_init(&raw_empty[s], kFConvWarps + (LP_TF32_RAW_HI ? 1 : 0));  // converter warps (+ the MMA commit)
    }
    for (int s = 0; s < kFCvStages; ++s) {
      mbar_init(&cv_full[s], 2 * kFConvWarps);  // converter warps x 2 CTAs (used in rank 0)
      mbar_init(&cv_empty[s], 1);   // leader's MMA commit (multicast)
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], 8);
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
  const int64_t ntiles = tiles.count();
  const int nkb = (int)(K / kFBK);

  if (warp == 0) {
    // ===================== TMA producer (both CTAs, own smem, own barrier) =====================
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int64_t t = pair; t < ntiles; t += npairs) {
        int64_t mb, nb;
        tiles.coords(t, mb, nb);
        const int m0 = (int)(mb * 256 + rank * 128), n0 = (int)(nb * 256 + rank * 128);
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&raw_empty[stage], phase ^ 1);
          mbar_expect_tx(&raw_full[stage], kFRawBytes);
          tma_load_2d(&tmap_a, &raw_full[stage], raw(stage), kb * kFBK, m0);
#pragma unroll
          for (int c = 0; c < 4; ++c)
            tma_load_2d(&tmap_b, &raw_full[stage], raw(stage) + kFTile + c * (kFBK * 128), n0 + c * 32, kb * kFBK);
          if (++stage == kFRawStages) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp >= kFConvWarp0) {
    // ===================== converters: raw -> [A_hi|A_lo|B_hi|B_lo] =====================
    const int ct = threadIdx.x - kFConvWarp0 * 32;  // 0 .. kFConvThreads - 1
    int rs = 0, cs = 0;
    uint32_t rphase = 0, cphase = 0;
    for (int64_t t = pair; t < ntiles; t += npairs) {
      for (int kb = 0; kb < nkb; ++kb) {
        mbar_wait(&raw_full[rs], rphase);
        mbar_wait(&cv_empty[cs], cphase ^ 1);
        const uint8_t* r = raw(rs);
        uint8_t* cv = cvs(cs);
        // A: K-major SW128 in and out -> element-wise over 1024 16-B units
#pragma unroll 4
        for (int i = ct; i < kFTile / 16; i += kFConvThreads) {
          const float4 x = *reinterpret_cast<const float4*>(r + i * 16);
          float4 hi, lo;
          hi.x = __uint_as_float(__float_as_uint(x.x) & 0xFFFFE000u);
          hi.y = __uint_as_float(__float_as_uint(x.y) & 0xFFFFE000u);
          hi.z = __uint_as_float(__float_as_uint(x.z) & 0xFFFFE000u);
          hi.w = __uint_as_float(__float_as_uint(x.w) & 0xFFFFE000u);
          lo.x = __fsub_rn(x.x, hi.x);
          lo.y = __fsub_rn(x.y, hi.y);
          lo.z = __fsub_rn(x.z, hi.z);
          lo.w = __fsub_rn(x.w, hi.w);
#if LP_TF32_RAW_HI_PROBE
          *reinterpret_cast<float4*>(cv + i * 16) = x;  // probe: the MMA reads the raw fp32 word as its tf32 hi
#elif !LP_TF32_RAW_HI
          *reinterpret_cast<float4*>(cv + i * 16) = hi;
#endif
          *reinterpret_cast<float4*>(cv + kFCvALo + i * 16) = lo;
        }
        // B: raw MN-major (chunk c = n/32 holds 32 K-rows x 32 columns, 16-B unit u of
        // row k stored at u ^ (k & 7)) -> K-major SW128 rows n (K quad j at j ^ (n & 7)).
        // Unit u = (column n = u % 128, K quad j = u / 128): the lanes of a warp read 32 consecutive columns
        // of one K row (conflict-free) and write 16-B units (optimal wavefronts).
        {
          // units (column n, K quad j): 128 x 8 per stage, strided over the converter threads
          // (LP_TF32_BLOOP=0: each thread takes consecutive K quads of one column, for 128 | 256 | 512 threads)
#if LP_TF32_BLOOP == 0
          constexpr int kJPer = (kFBK / 4) * 128 / kFConvThreads;
          static_assert(kJPer * kFConvThreads == (kFBK / 4) * 128, "column form needs 128, 256 or 512 threads");
#pragma unroll
          for (int jj = 0; jj < kJPer; ++jj) {
            const int n = ct & 127, j = (ct >> 7) * kJPer + jj, c = n >> 5, l = n & 31;
#else
#pragma unroll 2
          for (int u = ct; u < 128 * (kFBK / 4); u += kFConvThreads) {
            const int n = u & 127, j = u >> 7, c = n >> 5, l = n & 31;
#endif
            const uint8_t* rb = r + kFTile + c * (kFBK * 128) + (l & 3) * 4;
            uint8_t* bhi = cv + kFCvBHi + n * 128;
            uint8_t* blo = cv + kFCvBLo + n * 128;
            float xv[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const int k = 4 * j + e;
              xv[e] = *reinterpret_cast<const float*>(rb + k * 128 + (((l >> 2) ^ (k & 7)) << 4));
            }
            float4 hi, lo;
            hi.x = __uint_as_float(__float_as_uint(xv[0]) & 0xFFFFE000u);
            hi.y = __uint_as_float(__float_as_uint(xv[1]) & 0xFFFFE000u);
            hi.z = __uint_as_float(__float_as_uint(xv[2]) & 0xFFFFE000u);
            hi.w = __uint_as_float(__float_as_uint(xv[3]) & 0xFFFFE000u);
            lo.x = __fsub_rn(xv[0], hi.x);
            lo.y = __fsub_rn(xv[1], hi.y);
            lo.z = __fsub_rn(xv[2], hi.z);
            lo.w = __fsub_rn(xv[3], hi.w);
            const int off = ((j ^ (n & 7)) << 4);
#if LP_TF32_RAW_HI_PROBE
            *reinterpret_cast<float4*>(bhi + off) = make_float4(xv[0], xv[1], xv[2], xv[3]);
#else
            *reinterpret_cast<float4*>(bhi + off) = hi;
#endif
            *reinterpret_cast<float4*>(blo + off) = lo;
          }
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> tensor-core reads
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&raw_empty[rs]);
          if (rank == 0)
            mbar_arrive(&cv_full[cs]);
          else
            mbar_arrive_remote(mapa_rank0(&cv_full[cs]));
        }
        if (++rs == kFRawStages) {
          rs = 0;
          rphase ^= 1;
        }
        if (++cs == kFCvStages) {
          cs = 0;
          cphase ^= 1;
        }
      }
    }
  } else if (warp == 1) {
    // ===================== MMA issuer (leader, one thread) =====================
    if (lane == 0 && rank == 0) {
      // kind::tf32, D fp32, A and B both K-major, M = 256 (cta_group::2), N = 256
      constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (0u << 15) | (0u << 16) |
                                 ((uint32_t)(256 >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
      int stage = 0, rstage = 0;
      uint32_t phase = 0;
      uint32_t acc_phase = 0;
      for (int64_t t = pair; t < ntiles; t += npairs) {
        for (int kb0 = 0; kb0 < nkb; kb0 += chunk_kb) {
          const int kb1 = kb0 + chunk_kb < nkb ? kb0 + chunk_kb : nkb;
          mbar_wait(&tempty[0], acc_phase ^ 1);   // the epilogue has folded the previous chunk out of ACC
          tc_fence_after();
          const uint32_t d_tmem = tmem_base;       // ACC = TMEM columns [0, 256); SUM = [256, 512)
          for (int kb = kb0; kb < kb1; ++kb) {
            mbar_wait(&cv_full[stage], phase);
            tc_fence_after();
            const uint32_t cvb = smem_u32(cvs(stage));
            const uint32_t ah = LP_TF32_RAW_HI ? smem_u32(raw(rstage)) : cvb;  // raw A tile: K-major SW128 too
            const uint32_t al = cvb + kFCvALo, bh = cvb + kFCvBHi, bl = cvb + kFCvBLo;
#pragma unroll
            for (int k = 0; k < kFBK / kFUmmaK; ++k) {
              const uint64_t dah = smem_desc(ah + k * kFUmmaK * 4, 16, 1024);
              const uint64_t dal = smem_desc(al + k * kFUmmaK * 4, 16, 1024);
              const uint64_t dbh = smem_desc(bh + k * kFUmmaK * 4, 16, 1024);
              const uint64_t dbl = smem_desc(bl + k * kFUmmaK * 4, 16, 1024);
              tc_mma_pair_tf32(d_tmem, dah, dbh, idesc, (kb > kb0 || k > 0) ? 1u : 0u);
              tc_mma_pair_tf32(d_tmem, dah, dbl, idesc, 1u);
              tc_mma_pair_tf32(d_tmem, dal, dbh, idesc, 1u);
            }
            tc_commit_pair(&cv_empty[stage]);
            if (LP_TF32_RAW_HI) tc_commit_pair(&raw_empty[rstage]);   // the raw A tile is free once these MMAs ran
            if (++rstage == kFRawStages) rstage = 0;
            if (++stage == kFCvStages) {
              stage = 0;
              phase ^= 1;
            }
          }
          tc_commit_pair(&tfull[0]);  // this chunk's partial sum is ready
          acc_phase ^= 1;
        }
      }
    }
  } else {
    // ===================== epilogue (warps 2..5) =====================
    const int wq = warp & 3;
    uint32_t acc_phase = 0;
    int tile_iter = 0;
    for (int64_t t = pair; t < ntiles; t += npairs, ++tile_iter) {
      int64_t mb, nb;
      tiles.coords(t, mb, nb);
      const int64_t m128 = mb * 2 + rank;
      CkRecord* srec_acc = srec + (tile_iter & 1) * 2 * 4;   // per-tile double buffer of the warp partials
      const uint32_t t_acc = tmem_base + ((uint32_t)(wq * 32) << 16);
      const uint32_t t_sum = t_acc + (uint32_t)BN;
      for (int kb0 = 0; kb0 < nkb; kb0 += chunk_kb) {
        const bool first = kb0 == 0, last = kb0 + chunk_kb >= nkb;
        mbar_wait(&tfull[0], acc_phase);
        tc_fence_after();
        // SUM (+)= ACC in TMEM: IEEE fp32 adds in chunk order (Reading R22), then ACC goes back to the MMA
#pragma unroll 1
        for (int g = 0; g < BN / 32; ++g) {
          uint32_t r[32];
          LP_TMEM_LD32(t_acc + g * 32, r);
          if (!first) {
            uint32_t q[32];
            LP_TMEM_LD32(t_sum + g * 32, q);
            tc_wait_ld();
#pragma unroll
            for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(__fadd_rn(__uint_as_float(q[i]), __uint_as_float(r[i])));
          } else {
            tc_wait_ld();
          }
          LP_TMEM_ST32(t_sum + g * 32, r);
        }
        tc_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if (rank == 0)
            mbar_arrive(&tempty[0]);
          else
            mbar_arrive_remote(mapa_rank0(&tempty[0]));
        }
        if (last) {
          // C = SUM; the LP checksum is folded over exactly the stored words
          epi_store<float, MASK, REG, BN, STORE>(t_sum, C, ldc, m128, nb * BN, wq, lane, srec_acc, ck, tiles.Qr,
                                                 tiles.rid_offset, false, true);
          if constexpr (MASK != 0 && REG == 128)
            epi_finish_128<float, MASK, BN, STORE>(warp, lane, srec_acc, ck, m128, nb * BN, tiles.Qr,
                                                   tiles.rid_offset);
        }
        acc_phase ^= 1;
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

template <int REG>
cudaError_t launch_reg(const TmmArgs& a, cudaStream_t st, const char** why) {
  CUtensorMap ma, mb;
  if (!tma_map_2d(&ma, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.A, (uint64_t)a.K, (uint64_t)a.M, (uint64_t)a.lda, kFBK,
                  kBM, CU_TENSOR_MAP_SWIZZLE_128B) ||
      !tma_map_2d(&mb, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.B, (uint64_t)a.N, (uint64_t)a.K, (uint64_t)a.ldb, 32, kFBK,
                  CU_TENSOR_MAP_SWIZZLE_128B)) {
    *why = "cuTensorMapEncodeTiled failed";
    return cudaErrorInvalidValue;
  }
  PairTiles tl;
  tl.num_m = a.M / 256;
  tl.num_n = a.N / 256;
  tl.list = a.list;
  tl.d_n = a.d_n;
  tl.list_is_tiles = a.list_is_tiles;
  tl.Qr = a.N / REG;
  tl.rid_offset = a.rid_offset;
  tl.reg = REG;
  int64_t grid = a.list ? 2 * ((a.M / REG) * (a.N / REG)) : 2 * tl.num_m * tl.num_n;
  const int64_t cap = a.sm_count & ~1;
  if (grid > cap) grid = cap;
  if (grid < 2) grid = 2;
  const int sk = a.mask ? a.hash.store : 0;
  cudaError_t e = cudaSuccess;
  const int chunk_kb = kFChunkKB;
  switch (a.mask * 5 + sk) {
#define LP_TF_CASE(M, S)                                                                                    \
  case M * 5 + S: {                                                                                         \
    auto kfn = tmm_tf32x3_kernel<M, REG, S>;                                                               \
    e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, kFSmemBytes);                \
    if (e != cudaSuccess) return e;                                                                         \
    kfn<<<(unsigned)grid, kFThreads, kFSmemBytes, st>>>(ma, mb, (float*)a.C, a.ldc, a.K, tl, a.ck, chunk_kb); \
    break;                                                                                                  \
  }
#define LP_TF_CASE3(M) LP_TF_CASE(M, 0)
#define LP_TF_CASE5(M) LP_TF_CASE(M, 0) LP_TF_CASE(M, 1) LP_TF_CASE(M, 2) LP_TF_CASE(M, 3) LP_TF_CASE(M, 4)
    LP_TF_CASE(0, 0)
    LP_TF_CASE5(1)
    LP_TF_CASE3(2)
    LP_TF_CASE5(3)
    LP_TF_CASE3(4)
    LP_TF_CASE3(5)
    LP_TF_CASE3(6)
    LP_TF_CASE3(7)
#undef LP_TF_CASE3
#undef LP_TF_CASE5
#undef LP_TF_CASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace

bool tmm_tf32_supported(int64_t M, int64_t N, int64_t K, int RM, int RN, int in_bf16, int out_bf16, int64_t lda,
                        int64_t ldb, int64_t ldc, const void* A, const void* B, const void* C) {
  if (in_bf16 || out_bf16) return false;
  if (!((RM == 128 && RN == 128) || (RM == 32 && RN == 32))) return false;
  if (M % 256 || N % 256 || K % kFBK || K <= 0) return false;
  if ((lda * 4) % 16 || (ldb * 4) % 16 || (ldc * 4) % 16) return false;
  if ((((uintptr_t)A) & 15u) || (((uintptr_t)B) & 15u) || (((uintptr_t)C) & 15u)) return false;
  if (M > (int64_t)INT32_MAX || N > (int64_t)INT32_MAX || K > (int64_t)INT32_MAX) return false;
  return true;
}

cudaError_t launch_tmm_tf32(const TmmArgs& a, cudaStream_t st, const char** why) {
  return a.RM == 128 ? launch_reg<128>(a, st, why) : launch_reg<32>(a, st, why);
}

}  // namespace lp
