// spmv.cu -- LP-protected sparse matrix x dense vector region body (CSR), the
// paper's SPMV benchmark class (Table I: bandwidth-bound; Table IV
// L343: "SPMV go from just 22.1% to 437.6%" without warp shuffles).  NEXT row N4.
//
//   y[i] = sum_k p_k ,  p_k = fl(val[k] * x[col[k]])   (fp32, a fixed order per row: CSR order
//          for row pieces of <= 32 products per chunk, else lane-strided partials + butterfly)
//
// Region = region_n consecutive rows of y (1 x region_n block of the output
// vector viewed as [m / region_n][region_n]); one CTA per region, like the
// paper's thread-block regions (L181).  Idempotent (y is overwritten), so
// recovery re-runs the same code on the failed regions (L183).  The summation
// order of a row depends only on the row and its region's fixed chunk grid, so
// recovered rows are bit-identical by construction.
//
// Body (HBM-bound): the region's nnz range [rp[r0], rp[r0 + RN]) is contiguous in
// val[] and col[]; the CTA streams it in chunks of kChunk elements with 16-byte
// non-allocating loads (every thread 2 x (4 values + 4 columns) per chunk; the
// next chunk's loads are in flight while the current one is reduced), gathers
// x[col] through the read-only path (banded columns: L1/L2 hits), and writes the
// products into a double-buffered shared chunk.  Row phase: thread t owns rows
// ra + t, ra + t + 256, ... of the rows overlapping the chunk and adds the
// products of its row that fall in the chunk, in order, into the row's running
// sum (shared acc[]); pieces longer than 32 products are summed by a warp
// instead (fixed lane-strided order + butterfly).  The region's row_ptr slice is
// staged in shared memory once (relative int32 offsets).  (Measured: an 8-lane
// group per row, or 16-byte shared reads in the serial sums, were slower.)
//
// LP epilogue: y = acc is written coalesced and each thread folds the exact
// stored words of its rows into its checksum partials (L192, L260-261); warp
// redux.sync + a Listing-3 block combine give the region's record, stored
// lock-free at table[rid] (L349), or through the hash-store ablation.  SEQ =
// the paper's "no shuffle" ablation (L343): every thread's partials go through
// shared memory and thread 0 folds them sequentially.
#include <cuda_runtime.h>
#include <stdint.h>

#include "lp_device.cuh"
#include "lp_internal.h"

namespace lp {
namespace {

constexpr int kSpThreads = 256;
constexpr int kSpWarps = kSpThreads / 32;
#ifndef LP_SPMV_PT
#define LP_SPMV_PT 8
#endif
#ifndef LP_SPMV_MINB
#define LP_SPMV_MINB 5
#endif
#ifndef LP_SPMV_EARLY
#define LP_SPMV_EARLY 0
#endif
// element -> thread mapping of the product phase: 0 = each thread owns 4 consecutive elements per 16-B vector
// (lanes 4 elements apart: a warp's x gather touches ~32 lines of the banded x); 1 = element s*256 + tid
// (lanes on consecutive elements: ~8 lines per gather).  The shared product chunk, hence every sum, is the same.
#ifndef LP_SPMV_SCALAR
#define LP_SPMV_SCALAR 1
#endif
constexpr int kPerThread = LP_SPMV_PT;               // nnz per thread per chunk (kPerThread / 4 uint4)
constexpr int kVec = kPerThread / 4;
constexpr int kChunk = kSpThreads * kPerThread;      // nnz per chunk
constexpr int kLong = 32;                            // longer row pieces per chunk are summed by a warp

__device__ __forceinline__ uint4 ld_nc_u4(const void* p) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p));
  return r;
}

// Load this thread's 8 (value, column) pairs of the chunk starting at element kc
// (kc is 4-aligned; vectors entirely outside [K0, K1) are not loaded: value 0, column 0).
__device__ __forceinline__ void load_chunk(const float* __restrict__ val, const int32_t* __restrict__ col, int64_t kc,
                                           int64_t K0, int64_t K1, int64_t nnz, uint4* v, uint4* c) {
#pragma unroll
  for (int h = 0; h < kVec; ++h) {
    const int64_t k = kc + (int64_t)(h * kSpThreads + threadIdx.x) * 4;
    if (k + 4 > K0 && k < K1 && k + 4 <= nnz) {
      v[h] = ld_nc_u4(val + k);
      c[h] = ld_nc_u4(col + k);
    } else if (k + 4 > K0 && k < K1) {  // the array's last partial vector: element loads
      const uint32_t* vu = reinterpret_cast<const uint32_t*>(val);
      const uint32_t* cu = reinterpret_cast<const uint32_t*>(col);
      v[h].x = vu[k];
      c[h].x = cu[k];
      v[h].y = k + 1 < nnz ? vu[k + 1] : 0u;
      c[h].y = k + 1 < nnz ? cu[k + 1] : 0u;
      v[h].z = k + 2 < nnz ? vu[k + 2] : 0u;
      c[h].z = k + 2 < nnz ? cu[k + 2] : 0u;
      v[h].w = 0u;
      c[h].w = 0u;
    } else {
      v[h] = make_uint4(0u, 0u, 0u, 0u);
      c[h] = make_uint4(0u, 0u, 0u, 0u);
    }
  }
}

__device__ __forceinline__ uint32_t ld_nc_u32(const void* p) {
  uint32_t r;
  asm("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}

// Element kc + s * kSpThreads + tid of the chunk into slot s (0 outside [K0, K1)).
__device__ __forceinline__ void load_chunk_s(const float* __restrict__ val, const int32_t* __restrict__ col, int64_t kc,
                                             int64_t K0, int64_t K1, uint32_t* va, uint32_t* ca) {
#pragma unroll
  for (int s = 0; s < kPerThread; ++s) {
    const int64_t k = kc + (int64_t)s * kSpThreads + threadIdx.x;
    const bool in = k >= K0 && k < K1;
    va[s] = in ? ld_nc_u32(val + k) : 0u;
    ca[s] = in ? ld_nc_u32(col + k) : 0u;
  }
}

template <uint32_t MASK, int STORE, bool SEQ>
__global__ void __launch_bounds__(kSpThreads, LP_SPMV_MINB) spmv_kernel(const int64_t* __restrict__ row_ptr,
                                                          const int32_t* __restrict__ col,
                                                          const float* __restrict__ val,
                                                          const float* __restrict__ x, float* __restrict__ y,
                                                          int RN, int64_t R, int64_t n, int64_t nnz,
                                                          uint32_t* __restrict__ ck,
                                                          int64_t rid_offset, const int64_t* __restrict__ list,
                                                          const int64_t* __restrict__ d_n) {
  extern __shared__ __align__(16) uint8_t sm[];
  float* prod = reinterpret_cast<float*>(sm);                 // [2][kChunk]
  float* acc = prod + 2 * kChunk;                             // [RN]
  int32_t* srp = reinterpret_cast<int32_t*>(acc + RN);        // [RN + 1], relative to rp[r0]
  __shared__ CkRecord warp_rec[kSpWarps];
  __shared__ uint32_t seq_part[SEQ ? 4 : 1][SEQ ? kSpThreads : 1];
  __shared__ int s_ra, s_nlong;
  __shared__ int s_long[kChunk / (kLong + 1) + 1];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t ntiles = list ? *d_n : R;
  for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const int64_t rid = list ? (list[t] - rid_offset) : t;
    const int64_t r0 = rid * RN;  // first row of the region
    const int64_t K0 = row_ptr[r0], K1 = row_ptr[r0 + RN];
    for (int r = tid; r <= RN; r += kSpThreads) srp[r] = (int32_t)(row_ptr[r0 + r] - K0);
    for (int r = tid; r < RN; r += kSpThreads) acc[r] = 0.f;
    if (tid == 0) s_ra = 0;
    const int64_t kbase = K0 & ~(int64_t)3;
    const int nch = (int)((K1 - kbase + kChunk - 1) / kChunk);
#if LP_SPMV_SCALAR
    uint32_t va[kPerThread], ca[kPerThread];
    if (nch > 0) load_chunk_s(val, col, kbase, K0, K1, va, ca);
#else
    uint4 v[kVec], c[kVec];
    if (nch > 0) load_chunk(val, col, kbase, K0, K1, nnz, v, c);
#endif
    __syncthreads();
    for (int ch = 0; ch < nch; ++ch) {
      const int64_t kc = kbase + (int64_t)ch * kChunk;
      float* pb = prod + (ch & 1) * kChunk;
#if LP_SPMV_EARLY
      // the next chunk's (value, column) loads are issued before this chunk's x gathers, so HBM latency
      // overlaps the gathers, the products and the row phase
      uint4 vn[kVec], cn[kVec];
      if (ch + 1 < nch) load_chunk(val, col, kc + kChunk, K0, K1, nnz, vn, cn);
#endif
      // products of this thread's kPerThread elements (the x gathers are independent of each other);
      // masked lanes (value 0, column 0) read x[0] and store 0, never summed
      float xv[kPerThread];
#if LP_SPMV_SCALAR
#pragma unroll
      for (int e = 0; e < kPerThread; ++e) xv[e] = __ldg(x + (ca[e] < (uint64_t)n ? ca[e] : 0u));
#pragma unroll
      for (int e = 0; e < kPerThread; ++e) pb[e * kSpThreads + tid] = __fmul_rn(__uint_as_float(va[e]), xv[e]);
      if (ch + 1 < nch) load_chunk_s(val, col, kc + kChunk, K0, K1, va, ca);
#else
#pragma unroll
      for (int h = 0; h < kVec; ++h) {
        const uint32_t c4[4] = {c[h].x, c[h].y, c[h].z, c[h].w};
#pragma unroll
        for (int e = 0; e < 4; ++e) xv[4 * h + e] = __ldg(x + (c4[e] < (uint64_t)n ? c4[e] : 0u));
      }
#pragma unroll
      for (int h = 0; h < kVec; ++h) {
        float4 p;
        p.x = __fmul_rn(__uint_as_float(v[h].x), xv[4 * h + 0]);
        p.y = __fmul_rn(__uint_as_float(v[h].y), xv[4 * h + 1]);
        p.z = __fmul_rn(__uint_as_float(v[h].z), xv[4 * h + 2]);
        p.w = __fmul_rn(__uint_as_float(v[h].w), xv[4 * h + 3]);
        *reinterpret_cast<float4*>(pb + (h * kSpThreads + tid) * 4) = p;
      }
#if !LP_SPMV_EARLY
      // the next chunk's loads fly while this one is reduced
      if (ch + 1 < nch) load_chunk(val, col, kc + kChunk, K0, K1, nnz, v, c);
#endif
#if LP_SPMV_EARLY && !LP_SPMV_SCALAR
      if (ch + 1 < nch) {
#pragma unroll
        for (int h = 0; h < kVec; ++h) {
          v[h] = vn[h];
          c[h] = cn[h];
        }
      }
#endif
#endif  // LP_SPMV_SCALAR
      __syncthreads();
      // row phase: rows overlapping [lo, hi) (offsets relative to K0).  A row's products in this
      // chunk are summed in CSR order by its thread when there are <= kLong of them; longer
      // pieces (the heavy tail: up to a whole chunk) go to a warp -- lane-strided sequential
      // partials + a fixed xor butterfly -- so no chunk waits on one thread's long serial chain.
      // Either way the order is a fixed function of the row and the region's chunk grid.
      const int lo = (int)(kc - K0), hi = (int)(kc + kChunk - K0);
      const int ra = s_ra;
      if (tid == 0) s_nlong = 0;
      __syncthreads();  // everyone has read s_ra (and sees s_nlong = 0) before they change below
      for (int r = ra + tid; r < RN && srp[r] <= hi; r += kSpThreads) {
        const int b = srp[r] > lo ? srp[r] : lo;
        const int e = srp[r + 1] < hi ? srp[r + 1] : hi;
        if (e - b > kLong) {
          s_long[atomicAdd(&s_nlong, 1)] = r;
        } else if (b < e) {
          float s = acc[r];
          for (int k = b; k < e; ++k) s = __fadd_rn(s, pb[k - lo]);
          acc[r] = s;
        }
        if (hi < srp[r + 1]) s_ra = r;  // srp[r] <= hi < srp[r+1]: the row holding element hi
      }
      __syncthreads();
      for (int j = wid; j < s_nlong; j += kSpWarps) {
        const int r = s_long[j];
        const int b = srp[r] > lo ? srp[r] : lo;
        const int e = srp[r + 1] < hi ? srp[r + 1] : hi;
        float s = 0.f;
        for (int k = b + lane; k < e; k += 32) s = __fadd_rn(s, pb[k - lo]);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xFFFFFFFFu, s, o));
        if (lane == 0) acc[r] = __fadd_rn(acc[r], s);
      }
      // no barrier needed here: the next iteration writes the other product buffer, and its
      // first __syncthreads orders this row phase before this buffer is rewritten
    }
    __syncthreads();
    // y = acc, coalesced; fold the stored words (L192) -- 1-based byte position r*4 + 1
    CkPartial<MASK> part;
    for (int r = tid; r < RN; r += kSpThreads) {
      const float s = acc[r];
      y[r0 + r] = s;
      if constexpr (MASK != 0) part.add(__float_as_uint(s), (uint32_t)(r * 4 + 1));
    }
    if constexpr (MASK != 0) {
      if constexpr (SEQ) {
        seq_part[0][tid] = part.mod;
        seq_part[1][tid] = part.xr;
        seq_part[2][tid] = part.s;
        seq_part[3][tid] = (uint32_t)(part.w % kAdlerBase);
        __syncthreads();
        if (tid == 0) {
          CkRecord rr{0u, 0u, 0u, 0u};
          for (int j = 0; j < kSpThreads; ++j) {  // sequential, as on the CPU (L81, L220)
            rr.mod += seq_part[0][j];
            rr.xr ^= seq_part[1][j];
            rr.s += seq_part[2][j];
            rr.wmod = (rr.wmod + seq_part[3][j]) % kAdlerBase;
          }
          uint32_t words[3];
          record_words<MASK>(rr, (uint64_t)RN * 4, words);
          store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
        }
      } else {
        const CkRecord wr = warp_reduce<MASK>(part);
        if (lane == 0) warp_rec[wid] = wr;
        __syncthreads();
        if (tid == 0) {
          CkRecord rr = warp_rec[0];
#pragma unroll
          for (int w = 1; w < kSpWarps; ++w) rr = combine(rr, warp_rec[w]);
          uint32_t words[3];
          record_words<MASK>(rr, (uint64_t)RN * 4, words);
          store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
        }
      }
    }
    __syncthreads();  // shared state is reused by the next region of a persistent CTA
  }
}

size_t spmv_smem(int RN) { return (size_t)2 * kChunk * 4 + (size_t)RN * 4 + (size_t)(RN + 1) * 4; }

template <uint32_t MASK, int STORE>
cudaError_t launch_ms(const SpmvArgs& a, int64_t grid, int64_t R, cudaStream_t st) {
  const size_t smem = spmv_smem(a.RN);
  cudaError_t e;
  if (a.no_shuffle) {
    auto kfn = spmv_kernel<MASK, STORE, true>;
    if ((e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) != cudaSuccess) return e;
    kfn<<<(unsigned)grid, kSpThreads, smem, st>>>(a.row_ptr, a.col, a.val, a.x, a.y, a.RN, R, a.n, a.nnz, a.ck,
                                                  a.rid_offset, a.list, a.d_n);
  } else {
    auto kfn = spmv_kernel<MASK, STORE, false>;
    if ((e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) != cudaSuccess) return e;
    kfn<<<(unsigned)grid, kSpThreads, smem, st>>>(a.row_ptr, a.col, a.val, a.x, a.y, a.RN, R, a.n, a.nnz, a.ck,
                                                  a.rid_offset, a.list, a.d_n);
  }
  return cudaGetLastError();
}

}  // namespace

bool spmv_supported(int RN) { return RN >= 4 && RN <= 16384 && (RN & (RN - 1)) == 0; }

cudaError_t launch_spmv(const SpmvArgs& a, cudaStream_t st) {
  const int64_t R = a.m / a.RN;
  // full run: one region per CTA (the paper's TB = region); recovery: persistent CTAs over the list
  int64_t grid = a.list ? (R < (int64_t)a.sm_count * 8 ? R : (int64_t)a.sm_count * 8) : R;
  if (grid < 1) grid = 1;
  const int sk = a.mask ? a.hash.store : 0;
  switch (a.mask * 5 + sk) {
#define LP_SCASE(M, S) \
  case M * 5 + S:      \
    return launch_ms<M, S>(a, grid, R, st);
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
}

}  // namespace lp
