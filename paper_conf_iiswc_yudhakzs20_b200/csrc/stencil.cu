// stencil.cu -- LP-protected 5-point stencil region body (Reading R19).
//
// Stand-in for the paper's bandwidth-bound benchmark class (Table I:
// SPMV, SAD, HISTO), where the reduction's memory traffic hurts most (L343).
// Out-of-place, so each region is idempotent and recovery simply re-runs it
// (L183).  HBM-bound: 4 B read + 4 B written per output element.
//
//   out[i][j] = 0.5*in[i][j] + 0.125*(((in[i-1][j] + in[i+1][j]) + in[i][j-1]) + in[i][j+1])
//
// every op rounded to fp32 (__fadd_rn/__fmul_rn: no FMA contraction), zero
// outside the domain.  CTA = one 128x128 region; warp w owns 16 rows; each lane
// owns 4 adjacent columns (one 16-B vector).  All 18 input rows a lane needs
// are issued before any is used (18 x 16 B in flight per lane); the left/right
// neighbours come from the adjacent lanes through shuffles, the region's outer
// columns from one scalar load at each edge.  The checksum of the stored words
// is folded in registers (L192), warp-reduced with redux.sync and combined
// across the 8 warps in shared memory (Listings 3-4) before one thread stores
// the record at table[rid] (L349).
#include <cuda_runtime.h>
#include <stdint.h>

#include "lp_device.cuh"
#include "lp_internal.h"

namespace lp {
namespace {

constexpr int kRM = 128, kRN = 128;
constexpr int kWarps = 8;
constexpr int kRowsPerWarp = kRM / kWarps;  // 16

__device__ __forceinline__ float4 ld_row4(const float* in, int64_t ldi, int64_t H, int64_t i, int64_t j) {
  if (i < 0 || i >= H) return make_float4(0.f, 0.f, 0.f, 0.f);
  return __ldg(reinterpret_cast<const float4*>(in + i * ldi + j));
}

__device__ __forceinline__ float ld1(const float* in, int64_t ldi, int64_t H, int64_t W, int64_t i, int64_t j) {
  if (i < 0 || i >= H || j < 0 || j >= W) return 0.f;
  return __ldg(in + i * ldi + j);
}

__device__ __forceinline__ float st5(float c, float u, float d, float l, float r) {
  const float s = __fadd_rn(__fadd_rn(__fadd_rn(u, d), l), r);
  return __fadd_rn(__fmul_rn(0.5f, c), __fmul_rn(0.125f, s));
}

template <uint32_t MASK>
__global__ void __launch_bounds__(kWarps * 32) stencil5_kernel(const float* __restrict__ in, int64_t ldi,
                                                               float* __restrict__ out, int64_t ldo, int64_t H,
                                                               int64_t W, int64_t Q, int64_t R,
                                                               uint32_t* __restrict__ ck, int store,
                                                               int64_t rid_offset, const int64_t* __restrict__ list,
                                                               const int64_t* __restrict__ d_n) {
  __shared__ CkRecord warp_rec[kWarps];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t ntiles = list ? *d_n : R;
  for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const int64_t rid = list ? (list[t] - rid_offset) : t;
    const int64_t p = rid / Q, q = rid - p * Q;
    const int64_t i0 = p * kRM + wid * kRowsPerWarp;
    const int64_t j = q * kRN + lane * 4;

    float4 v[kRowsPerWarp + 2];
#pragma unroll
    for (int r = 0; r < kRowsPerWarp + 2; ++r) v[r] = ld_row4(in, ldi, H, i0 - 1 + r, j);
    float edge[kRowsPerWarp];
#pragma unroll
    for (int r = 0; r < kRowsPerWarp; ++r) {
      // lane 0 needs column j-1, lane 31 needs column j+4 (outside this warp's 128 columns)
      edge[r] = lane == 0 ? ld1(in, ldi, H, W, i0 + r, j - 1) : (lane == 31 ? ld1(in, ldi, H, W, i0 + r, j + 4) : 0.f);
    }

    CkPartial<MASK> part;
#pragma unroll
    for (int r = 0; r < kRowsPerWarp; ++r) {
      const float4 u = v[r], c = v[r + 1], d = v[r + 2];
      float left = __shfl_up_sync(0xFFFFFFFFu, c.w, 1);
      float right = __shfl_down_sync(0xFFFFFFFFu, c.x, 1);
      if (lane == 0) left = edge[r];
      if (lane == 31) right = edge[r];
      float4 o;
      o.x = st5(c.x, u.x, d.x, left, c.y);
      o.y = st5(c.y, u.y, d.y, c.x, c.z);
      o.z = st5(c.z, u.z, d.z, c.y, c.w);
      o.w = st5(c.w, u.w, d.w, c.z, right);
      *reinterpret_cast<float4*>(out + (i0 + r) * ldo + j) = o;
      if constexpr (MASK != 0) {
        const uint32_t pos = (uint32_t)((wid * kRowsPerWarp + r) * kRN * 4 + lane * 16 + 1);
        part.add(__float_as_uint(o.x), pos);
        part.add(__float_as_uint(o.y), pos + 4);
        part.add(__float_as_uint(o.z), pos + 8);
        part.add(__float_as_uint(o.w), pos + 12);
      }
    }
    if constexpr (MASK != 0) {
      const CkRecord wr = warp_reduce<MASK>(part);
      if (lane == 0) warp_rec[wid] = wr;
      __syncthreads();
      if (threadIdx.x == 0) {
        CkRecord rr = warp_rec[0];
#pragma unroll
        for (int w = 1; w < kWarps; ++w) rr = combine(rr, warp_rec[w]);
        uint32_t words[3];
        record_words<MASK>(rr, (uint64_t)kRM * kRN * 4, words);
        store_record<MASK>(ck, store, rid, (uint32_t)(rid + rid_offset), words);
      }
      __syncthreads();
    }
  }
}

}  // namespace

bool stencil_supported(int RM, int RN) { return RM == kRM && RN == kRN; }

cudaError_t launch_stencil(const StencilArgs& a, cudaStream_t st) {
  const int64_t Q = a.W / kRN, R = (a.H / kRM) * Q;
  int64_t grid = a.list ? (int64_t)a.sm_count * 8 : R;
  if (a.list && grid > R) grid = R;
  if (grid < 1) grid = 1;
  switch (a.mask) {
#define LP_TCASE(M)                                                                                            \
  case M:                                                                                                      \
    stencil5_kernel<M><<<(unsigned)grid, kWarps * 32, 0, st>>>(a.in, a.ldi, a.out, a.ldo, a.H, a.W, Q, R, a.ck, \
                                                               a.hash.store, a.rid_offset, a.list, a.d_n);     \
    break;
    LP_TCASE(0)
    LP_TCASE(1)
    LP_TCASE(2)
    LP_TCASE(3)
    LP_TCASE(4)
    LP_TCASE(5)
    LP_TCASE(6)
    LP_TCASE(7)
#undef LP_TCASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace lp
