// tmm_simt.cu -- SIMT LP-protected tiled matrix multiply, paper-shaped.
//
// The paper's TMM (Listing 2; Listing 6) is a SIMT kernel
// whose thread block computes one output tile through shared-memory A/B tiles
// and is the LP region (L181 §IV-A).  This is that design on sm_100a, kept as
// the prior-art body (and the fp32-input body): CTA tile == region, 256
// threads with a register micro-tile, fp32 FFMA accumulate, K in fixed order
// (deterministic: recovery reproduces the golden bits, Reading R18).
//
// LP epilogue (fused, no extra pass over C): every thread folds the exact
// 32-bit words it stores into its checksum partials (L192), the warp reduces
// them with one redux.sync per checksum (Listing 4 L244-258 -> redux), warps
// combine through shared memory (Listing 3), and one thread stores
// the record lock-free at table[rid] (L349 §V).
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "lp_device.cuh"
#include "lp_internal.h"
#include "lp_ptx.cuh"

namespace lp {
namespace {

constexpr int kThreads = 256;
// CTAs per SM the 128x128-tile builds are compiled for (1: ptxas takes ~240 registers; 2: <= 128)
#ifndef LP_SIMT_MINB
#define LP_SIMT_MINB 2
#endif
#ifndef LP_SIMT_ASYNC
#define LP_SIMT_ASYNC 1
#endif
constexpr int kBK = 16;

// compute type: fp32 for float / bf16 operands (FFMA), int32 for the paper's int TMM (IMAD, wrapping)
template <typename T>
struct Acc {
  using type = float;
};
template <>
struct Acc<int32_t> {
  using type = int32_t;
};
template <typename T>
__device__ __forceinline__ typename Acc<T>::type to_acc(T v) {
  return v;
}
template <>
__device__ __forceinline__ float to_acc<__nv_bfloat16>(__nv_bfloat16 v) {
  return __bfloat162float(v);
}
__device__ __forceinline__ float mac(float a, float b, float c) { return fmaf(a, b, c); }
__device__ __forceinline__ int32_t mac(int32_t a, int32_t b, int32_t c) {
  return (int32_t)((uint32_t)a * (uint32_t)b + (uint32_t)c);
}
// Fragment loads from shared memory, explicitly vectorised so the protected kernel
// and its unprotected twin compile to the same mainloop (the overhead denominator).
template <int U, typename TA>
__device__ __forceinline__ void load_frag(TA* dst, const TA* src) {
  static_assert(sizeof(TA) == 4, "32-bit compute types");
  if constexpr (U % 4 == 0) {
#pragma unroll
    for (int i = 0; i < U; i += 4) *reinterpret_cast<uint4*>(dst + i) = *reinterpret_cast<const uint4*>(src + i);
  } else if constexpr (U % 2 == 0) {
#pragma unroll
    for (int i = 0; i < U; i += 2) *reinterpret_cast<uint2*>(dst + i) = *reinterpret_cast<const uint2*>(src + i);
  } else {
#pragma unroll
    for (int i = 0; i < U; ++i) dst[i] = src[i];
  }
}

template <typename T>
__device__ __forceinline__ uint32_t word_of(T v);
template <>
__device__ __forceinline__ uint32_t word_of<float>(float v) { return __float_as_uint(v); }
template <>
__device__ __forceinline__ uint32_t word_of<int32_t>(int32_t v) { return (uint32_t)v; }

// SEQ = the paper's "no shuffle" ablation (L343, Table IV "+no"): partials go to
// shared memory and ONE thread folds all 256 of them sequentially, O(N) instead of
// the O(log N) warp reduction (L220).
// RMR x RNR = the LP region.  RMR == BM, RNR == BN: the CTA tile is the region (the paper's TB = region,
// L181).  Smaller regions (the paper's 32x32, Table V TMM) may tile a 128x128 CTA tile (Reading c10): every
// thread's UM x UN micro-tile lies inside one region, the region's partials are combined by a segmented xor
// butterfly inside the warp and a two-warp combine through shared memory, and one record per region is
// stored -- 16 records per CTA, with the 8x8 register micro-tiles of the 128x128 tile instead of 2x2.
template <typename TIn, typename TOut, int BM, int BN, int UM, int UN, uint32_t MASK, int STORE, bool SEQ = false,
          int RMR = BM, int RNR = BN>
__global__ void __launch_bounds__(kThreads, (BM * BN >= 128 * 128) ? LP_SIMT_MINB : 1) tmm_simt_kernel(const TIn* __restrict__ A, int64_t lda,
                                                            const TIn* __restrict__ B, int64_t ldb,
                                                            TOut* __restrict__ C, int64_t ldc, int64_t K,
                                                            int64_t Q, int64_t R, uint32_t* __restrict__ ck,
                                                            int64_t rid_offset,
                                                            const int64_t* __restrict__ list,
                                                            const int64_t* __restrict__ d_n) {
  static_assert((BM / UM) * (BN / UN) == kThreads, "256 threads");
  static_assert(UN % 2 == 0, "bf16 words pair two columns");
  constexpr int TX = BN / UN;  // threads along N
  constexpr int A_PER = BM * kBK / kThreads;
  constexpr int B_PER = BN * kBK / kThreads;
  static_assert(A_PER >= 1 && B_PER >= 1, "tile too small");
  constexpr int ES = (int)sizeof(TOut);
  using TA = typename Acc<TIn>::type;

  __shared__ __align__(16) TA As[2][kBK][BM + 4];
  __shared__ __align__(16) TA Bs[2][kBK][BN + 4];
  constexpr bool kMulti = RMR != BM || RNR != BN;
  __shared__ CkRecord warp_rec[kMulti ? (kThreads / 32) * (BN / RNR) : kThreads / 32];
  __shared__ uint32_t seq_part[SEQ ? 4 : 1][SEQ ? kThreads : 1];

  const int tid = threadIdx.x;
  const int tx = tid % TX, ty = tid / TX;

  const int64_t ntiles = list ? *d_n : R;
  for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const int64_t rid = list ? (list[t] - rid_offset) : t;
    const int64_t p = rid / Q, q = rid - p * Q;
    const int64_t row0 = p * BM, col0 = q * BN;

    TA acc[UM][UN];
#pragma unroll
    for (int i = 0; i < UM; ++i)
#pragma unroll
      for (int j = 0; j < UN; ++j) acc[i][j] = TA(0);

    // 4-byte operands that need no conversion (fp32, int32) go global -> shared with cp.async (no register
    // staging: the 128x128 builds then fit 2 CTAs/SM without spills); bf16 is converted through registers
    constexpr bool kAsync = sizeof(TIn) == 4 && LP_SIMT_ASYNC;
    auto aload = [&](int64_t k0, int buf) {
#pragma unroll
      for (int i = 0; i < A_PER; ++i) {
        const int e = tid + i * kThreads;
        const int m = e / kBK, k = e % kBK;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(&As[buf][k][m])),
                     "l"(A + (row0 + m) * lda + k0 + k) : "memory");
      }
#pragma unroll
      for (int i = 0; i < B_PER; ++i) {
        const int e = tid + i * kThreads;
        const int k = e / BN, n = e % BN;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(&Bs[buf][k][n])),
                     "l"(B + (k0 + k) * ldb + col0 + n) : "memory");
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    };
    TA ra[kAsync ? 1 : A_PER], rb[kAsync ? 1 : B_PER];
    auto gload = [&](int64_t k0) {
#pragma unroll
      for (int i = 0; i < A_PER; ++i) {
        const int e = tid + i * kThreads;
        const int m = e / kBK, k = e % kBK;
        ra[i] = to_acc(A[(row0 + m) * lda + k0 + k]);
      }
#pragma unroll
      for (int i = 0; i < B_PER; ++i) {
        const int e = tid + i * kThreads;
        const int k = e / BN, n = e % BN;
        rb[i] = to_acc(B[(k0 + k) * ldb + col0 + n]);
      }
    };
    auto sstore = [&](int buf) {
#pragma unroll
      for (int i = 0; i < A_PER; ++i) {
        const int e = tid + i * kThreads;
        As[buf][e % kBK][e / kBK] = ra[i];
      }
#pragma unroll
      for (int i = 0; i < B_PER; ++i) {
        const int e = tid + i * kThreads;
        Bs[buf][e / BN][e % BN] = rb[i];
      }
    };

    __syncthreads();  // previous tile's smem readers are done
    if constexpr (kAsync) {
      aload(0, 0);
      asm volatile("cp.async.wait_all;" ::: "memory");
    } else {
      gload(0);
      sstore(0);
    }
    __syncthreads();
    const int64_t nk = K / kBK;
    for (int64_t kt = 0; kt < nk; ++kt) {
      const int buf = (int)(kt & 1);
      if constexpr (kAsync) {
        if (kt + 1 < nk) aload((kt + 1) * kBK, buf ^ 1);  // buf ^ 1 was released by the previous barrier
      } else {
        if (kt + 1 < nk) gload((kt + 1) * kBK);
      }
#pragma unroll
      for (int k = 0; k < kBK; ++k) {
        TA a[UM], b[UN];
        load_frag<UM>(a, &As[buf][k][ty * UM]);
        load_frag<UN>(b, &Bs[buf][k][tx * UN]);
#pragma unroll
        for (int i = 0; i < UM; ++i)
#pragma unroll
          for (int j = 0; j < UN; ++j) acc[i][j] = mac(a[i], b[j], acc[i][j]);
      }
      if constexpr (kAsync) {
        asm volatile("cp.async.wait_all;" ::: "memory");
      } else {
        if (kt + 1 < nk) sstore(buf ^ 1);
      }
      __syncthreads();
    }

    // ---- epilogue: store + checksum over the exact stored words
    CkPartial<MASK> part;
#pragma unroll
    for (int i = 0; i < UM; ++i) {
      const int lr = ty * UM + i;
      TOut* crow = C + (row0 + lr) * ldc + col0 + tx * UN;
#pragma unroll
      for (int j = 0; j < UN; j += 2) {
        uint32_t w0, w1 = 0;
        if constexpr (ES == 4) {
          const TOut o0 = (TOut)acc[i][j], o1 = (TOut)acc[i][j + 1];
          w0 = word_of<TOut>(o0);
          w1 = word_of<TOut>(o1);
          *reinterpret_cast<uint2*>(crow + j) = make_uint2(w0, w1);
        } else {
          __nv_bfloat162 h = __floats2bfloat162_rn(acc[i][j], acc[i][j + 1]);  // .x (even col) -> low half
          w0 = *reinterpret_cast<uint32_t*>(&h);
          *reinterpret_cast<__nv_bfloat162*>(crow + j) = h;
        }
        if constexpr (MASK != 0) {
          const uint32_t pos = (uint32_t)((lr % RMR) * RNR * ES + ((tx * UN + j) % RNR) * ES + 1);
          part.add(w0, pos);
          if constexpr (ES == 4) part.add(w1, pos + 4);
        }
      }
    }
    if constexpr (MASK != 0 && kMulti && SEQ) {
      // the no-shuffle ablation (L343) on the multi-region tile: every thread parks its partials in shared
      // memory and ONE thread per region folds its region's 16 threads' partials sequentially
      static_assert(BM == 128 && BN == 128 && UM == 8 && UN == 8 && RMR == 32 && RNR == 32, "one multi-region shape");
      seq_part[0][tid] = part.mod;
      seq_part[1][tid] = part.xr;
      seq_part[2][tid] = part.s;
      seq_part[3][tid] = (uint32_t)(part.w % kAdlerBase);
      __syncthreads();
      if (tid < 16) {
        const int ry = tid >> 2, rx = tid & 3;
        CkRecord rr{0u, 0u, 0u, 0u};
        for (int ty2 = 4 * ry; ty2 < 4 * ry + 4; ++ty2)
          for (int tx2 = 4 * rx; tx2 < 4 * rx + 4; ++tx2) {
            const int j = ty2 * 16 + tx2;
            rr.mod += seq_part[0][j];
            rr.xr ^= seq_part[1][j];
            rr.s += seq_part[2][j];
            rr.wmod = (rr.wmod + seq_part[3][j]) % kAdlerBase;
          }
        uint32_t words[3];
        record_words<MASK>(rr, (uint64_t)RMR * RNR * ES, words);
        const int64_t rrid = (p * 4 + ry) * (Q * 4) + q * 4 + rx;
        store_record<MASK, STORE>(ck, rrid, (uint32_t)(rrid + rid_offset), words);
      }
    } else if constexpr (MASK != 0 && kMulti) {
      // 128x128 tile, 8x8 micro-tiles, 32x32 regions: a warp = 2 rows of threads (ty) x 16 columns (tx); the
      // 4 x 4 threads of a region are lanes {4a..4a+3} x {+0, +16} of two consecutive warps
      static_assert(BM == 128 && BN == 128 && UM == 8 && UN == 8 && RMR == 32 && RNR == 32, "one multi-region shape");
      CkRecord r{part.mod, part.xr, part.s, 0u};
      if constexpr ((MASK & kAdler) != 0) r.wmod = (uint32_t)(part.w % kAdlerBase);
#pragma unroll
      for (int o : {1, 2, 16}) {
        if constexpr ((MASK & kMod) != 0) r.mod += __shfl_xor_sync(0xFFFFFFFFu, r.mod, o);
        if constexpr ((MASK & kXor) != 0) r.xr ^= __shfl_xor_sync(0xFFFFFFFFu, r.xr, o);
        if constexpr ((MASK & kAdler) != 0) {
          r.s += __shfl_xor_sync(0xFFFFFFFFu, r.s, o);
          r.wmod += __shfl_xor_sync(0xFFFFFFFFu, r.wmod, o);
        }
      }
      const int lane = tid & 31, warp = tid >> 5;
      if ((lane & 19) == 0) warp_rec[warp * 4 + (lane >> 2)] = r;  // lanes 0, 4, 8, 12: region column lane / 4
      __syncthreads();
      if (tid < 16) {
        const int ry = tid >> 2, rx = tid & 3;
        const CkRecord rr = combine(warp_rec[(2 * ry) * 4 + rx], warp_rec[(2 * ry + 1) * 4 + rx]);
        uint32_t words[3];
        record_words<MASK>(rr, (uint64_t)RMR * RNR * ES, words);
        const int64_t rrid = (p * 4 + ry) * (Q * 4) + q * 4 + rx;  // region id in the 32x32 grid
        store_record<MASK, STORE>(ck, rrid, (uint32_t)(rrid + rid_offset), words);
      }
    } else if constexpr (MASK != 0 && SEQ) {
      seq_part[0][tid] = part.mod;
      seq_part[1][tid] = part.xr;
      seq_part[2][tid] = part.s;
      seq_part[3][tid] = (uint32_t)(part.w % kAdlerBase);
      __syncthreads();
      if (tid == 0) {
        CkRecord r{0u, 0u, 0u, 0u};
        for (int i = 0; i < kThreads; ++i) {  // sequential, as on the CPU (L81, L220)
          r.mod += seq_part[0][i];
          r.xr ^= seq_part[1][i];
          r.s += seq_part[2][i];
          r.wmod = (r.wmod + seq_part[3][i]) % kAdlerBase;
        }
        uint32_t words[3];
        record_words<MASK>(r, (uint64_t)BM * BN * ES, words);
        store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
      }
    } else if constexpr (MASK != 0) {
      const CkRecord wr = warp_reduce<MASK>(part);
      if ((tid & 31) == 0) warp_rec[tid >> 5] = wr;
      __syncthreads();
      if (tid == 0) {
        CkRecord r = warp_rec[0];
#pragma unroll
        for (int w = 1; w < kThreads / 32; ++w) r = combine(r, warp_rec[w]);
        uint32_t words[3];
        record_words<MASK>(r, (uint64_t)BM * BN * ES, words);
        store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
      }
    }
  }
}

template <typename TIn, typename TOut, int BM, int BN, int UM, int UN>
cudaError_t launch_mask(const TmmArgs& a, cudaStream_t st) {
  const int64_t Q = a.N / BN, R = (a.M / BM) * Q;
  int64_t grid = a.list ? (int64_t)a.sm_count * 4 : R;
  if (a.list && grid > R) grid = R;
  if (grid < 1) grid = 1;
  const TIn* A = (const TIn*)a.A;
  const TIn* B = (const TIn*)a.B;
  TOut* C = (TOut*)a.C;
  const int sk = a.mask ? a.hash.store : 0;
  if (a.no_shuffle) {
    if (a.mask != 3) return cudaErrorInvalidValue;  // the ablation is built for MOD|XOR (Table IV)
    switch (sk) {
#define LP_QCASE(S)                                                                                            \
  case S:                                                                                                      \
    tmm_simt_kernel<TIn, TOut, BM, BN, UM, UN, 3, S, true><<<(unsigned)grid, kThreads, 0, st>>>(               \
        A, a.lda, B, a.ldb, C, a.ldc, a.K, Q, R, a.ck, a.rid_offset, a.list, a.d_n);                           \
    break;
      LP_QCASE(0)
      LP_QCASE(1)
      LP_QCASE(2)
      LP_QCASE(3)
      LP_QCASE(4)
#undef LP_QCASE
      default:
        return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
  }
  switch (a.mask * 5 + sk) {
#define LP_SCASE(M, S)                                                                                         \
  case M * 5 + S:                                                                                              \
    tmm_simt_kernel<TIn, TOut, BM, BN, UM, UN, M, S><<<(unsigned)grid, kThreads, 0, st>>>(                     \
        A, a.lda, B, a.ldb, C, a.ldc, a.K, Q, R, a.ck, a.rid_offset, a.list, a.d_n);                           \
    break;
#define LP_SCASE3(M) LP_SCASE(M, 0)
#define LP_SCASE5(M) LP_SCASE(M, 0) LP_SCASE(M, 1) LP_SCASE(M, 2) LP_SCASE(M, 3) LP_SCASE(M, 4)
    LP_SCASE(0, 0)
    LP_SCASE5(1)
    LP_SCASE3(2)
    LP_SCASE5(3)
    LP_SCASE3(4)
    LP_SCASE3(5)
    LP_SCASE3(6)
    LP_SCASE3(7)
#undef LP_SCASE3
#undef LP_SCASE5
#undef LP_SCASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

// full runs of 32x32 regions on 128x128 CTA tiles (16 regions per tile; the no-shuffle ablation too);
// list-mode recovery and shapes not divisible by 128 keep one CTA per 32x32 region
template <typename TIn, typename TOut>
cudaError_t launch_multi32(const TmmArgs& a, cudaStream_t st) {
  const int64_t Q = a.N / 128, R = (a.M / 128) * Q;
  const TIn* A = (const TIn*)a.A;
  const TIn* B = (const TIn*)a.B;
  TOut* C = (TOut*)a.C;
  const int sk = a.mask ? a.hash.store : 0;
  if (a.no_shuffle) {
    if (a.mask != 3) return cudaErrorInvalidValue;  // the ablation is built for MOD|XOR (Table IV)
    switch (sk) {
#define LP_MQCASE(S)                                                                                           \
  case S:                                                                                                      \
    tmm_simt_kernel<TIn, TOut, 128, 128, 8, 8, 3, S, true, 32, 32><<<(unsigned)R, kThreads, 0, st>>>(           \
        A, a.lda, B, a.ldb, C, a.ldc, a.K, Q, R, a.ck, a.rid_offset, nullptr, nullptr);                         \
    break;
      LP_MQCASE(0)
      LP_MQCASE(1)
      LP_MQCASE(2)
      LP_MQCASE(3)
      LP_MQCASE(4)
#undef LP_MQCASE
      default:
        return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
  }
  switch (a.mask * 5 + sk) {
#define LP_MCASE(M, S)                                                                                         \
  case M * 5 + S:                                                                                              \
    tmm_simt_kernel<TIn, TOut, 128, 128, 8, 8, M, S, false, 32, 32><<<(unsigned)R, kThreads, 0, st>>>(          \
        A, a.lda, B, a.ldb, C, a.ldc, a.K, Q, R, a.ck, a.rid_offset, nullptr, nullptr);                         \
    break;
#define LP_MCASE3(M) LP_MCASE(M, 0)
#define LP_MCASE5(M) LP_MCASE(M, 0) LP_MCASE(M, 1) LP_MCASE(M, 2) LP_MCASE(M, 3) LP_MCASE(M, 4)
    LP_MCASE(0, 0)
    LP_MCASE5(1)
    LP_MCASE3(2)
    LP_MCASE5(3)
    LP_MCASE3(4)
    LP_MCASE3(5)
    LP_MCASE3(6)
    LP_MCASE3(7)
#undef LP_MCASE3
#undef LP_MCASE5
#undef LP_MCASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

bool simt_multi32() {
  static bool v = [] {
    const char* e = getenv("LP_SIMT_MULTI");
    return e ? atoi(e) != 0 : true;
  }();
  return v;
}

template <typename TIn, typename TOut>
cudaError_t launch_shape(const TmmArgs& a, cudaStream_t st) {
  if (a.RM == 32 && a.RN == 32 && !a.list && a.M % 128 == 0 && a.N % 128 == 0 && simt_multi32())
    return launch_multi32<TIn, TOut>(a, st);
  if (a.RM == 32 && a.RN == 32) return launch_mask<TIn, TOut, 32, 32, 2, 2>(a, st);
  if (a.RM == 64 && a.RN == 64) return launch_mask<TIn, TOut, 64, 64, 4, 4>(a, st);
  if (a.RM == 128 && a.RN == 128) return launch_mask<TIn, TOut, 128, 128, 8, 8>(a, st);
  return cudaErrorInvalidValue;
}

}  // namespace

bool tmm_simt_supported(int RM, int RN, int, int) {
  return (RM == 32 && RN == 32) || (RM == 64 && RN == 64) || (RM == 128 && RN == 128);
}

cudaError_t launch_tmm_simt(const TmmArgs& a, cudaStream_t st) {
  if (a.i32) return launch_shape<int32_t, int32_t>(a, st);
  if (a.in_bf16) {
    return a.out_bf16 ? launch_shape<__nv_bfloat16, __nv_bfloat16>(a, st) : launch_shape<__nv_bfloat16, float>(a, st);
  }
  return a.out_bf16 ? launch_shape<float, __nv_bfloat16>(a, st) : launch_shape<float, float>(a, st);
}

}  // namespace lp
