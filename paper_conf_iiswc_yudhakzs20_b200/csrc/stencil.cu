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
// outside the domain.
//
// Structure: CTA = one 128x128 region, 8 warps x 16 rows, lane = 4 adjacent
// columns (one 16-B vector).  Every lane issues all 18 row loads and its edge
// loads up front (non-allocating 16-B loads through volatile PTX), then
// computes; left/right neighbours come from the adjacent lanes by shuffle;
// results leave with streaming 16-B stores.  2 CTAs (16 warps) per SM.
// Protected full runs use the two-phase epilogue: the 16 edge values of a warp
// are loaded one per lane (lanes 0-15 left, 16-31 right) and broadcast by
// shuffle, every row is stored first, and the checksum pass runs over the
// stored vectors afterwards (four Adler accumulator sets); the plain twin keeps
// per-row edge loads, its fastest form (A/B in profiles/r02/ab_stencil_epilogue.txt).
//
// LP epilogue: each lane folds the exact stored words into its checksum
// partials (L192) and the warp reduces them with redux.sync (Listing 4).  The
// 8 warps' partials are combined behind a SPLIT barrier: every warp parks its
// partial in shared memory and arrives (bar.arrive) on a named barrier; only
// warp 0 waits (bar.sync), combines (Listing 3) and stores the record at
// table[rid] (L349).  The unprotected twin keeps the same barrier (it also
// speeds the plain kernel up), so the LP overhead compares like with like.
// (List-mode recovery, where a CTA handles several regions, uses the barrier
// combine; measured A/Bs in DESIGN.md.)
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "lp_device.cuh"
#include "lp_internal.h"
#include "lp_ptx.cuh"
#include "lp_tma.h"

namespace lp {
namespace {

constexpr int kRM = 128, kRN = 128;
#ifndef LP_STENCIL_TWIN_BAR
#define LP_STENCIL_TWIN_BAR 1
#endif

__device__ __forceinline__ float st5(float c, float u, float d, float l, float r) {
  const float s = __fadd_rn(__fadd_rn(__fadd_rn(u, d), l), r);
  return __fadd_rn(__fmul_rn(0.5f, c), __fmul_rn(0.125f, s));
}

// Adler-32 partials of one lane's column of 16-byte vectors, one vector per region row (kRowsW rows, row
// pitch row_bytes inside the region's byte stream).  Instead of a 64-bit position multiply per vector
// (CkPartial::add4), the row index is folded in with a running-sum trick: S chains the byte sums through
// dp4a, T accumulates S after every row (T = sum_r (n - r) * bs_r), Wl chains the in-vector weights
// 0..15 through dp4a; then  W = base * S + row_bytes * (n * S - T) + Wl  with base = the 1-based stream
// position of this lane's first byte.  Exactly the sums of add4 (integer arithmetic), 9 ops per row.
struct AdlerRows {
  uint32_t S = 0, T = 0, Wl = 0;
  __device__ __forceinline__ void add_row(uint32_t x, uint32_t y, uint32_t z, uint32_t v) {
    S = (uint32_t)__dp4a(x, 0x01010101u, __dp4a(y, 0x01010101u, __dp4a(z, 0x01010101u, __dp4a(v, 0x01010101u, S))));
    Wl = (uint32_t)__dp4a(x, 0x03020100u, __dp4a(y, 0x07060504u, __dp4a(z, 0x0B0A0908u, __dp4a(v, 0x0F0E0D0Cu, Wl))));
    T += S;
  }
  template <uint32_t MASK>
  __device__ __forceinline__ void fold(CkPartial<MASK>& p, uint32_t base, uint32_t nrows, uint32_t row_bytes) const {
    p.s += S;
    p.w += (uint64_t)base * S + (uint64_t)row_bytes * (uint64_t)(nrows * S - T) + Wl;
  }
};

// MOD / XOR part of CkPartial::add4 (the Adler part goes through AdlerRows)
template <uint32_t MASK>
__device__ __forceinline__ void add4_modxor(CkPartial<MASK>& p, uint32_t x, uint32_t y, uint32_t z, uint32_t v) {
  if constexpr ((MASK & kMod) != 0) p.mod += (x + y) + (z + v);
  if constexpr ((MASK & kXor) != 0) p.xr ^= x ^ y ^ z ^ v;
}

// output stores of the LDG form: the two-phase protected kernels with Adler in the record store with .cg (cache
// at L2), the others (MOD / XOR, and the plain twin) with evict-first .cs -- each its faster flavour
// (profiles/r02/ab_stencil_st.txt: Adler 1.330 -> 1.314 ms with .cg; the twin 1.300 with .cs vs 1.304-1.308;
// MOD|XOR equal); LP_STENCIL_ST=1..3 force one flavour everywhere (A/B runs)
#ifndef LP_STENCIL_ST
#define LP_STENCIL_ST 0
#endif
#ifndef LP_STENCIL_TMA_ST_CG  // TMA-fed form (list-mode recovery): .cg instead of .cs output stores
#define LP_STENCIL_TMA_ST_CG 0
#endif
template <bool CG>
__device__ __forceinline__ void st_out(float4* p, float4 o) {
#if LP_STENCIL_ST == 0
  if constexpr (CG) {
    asm volatile("st.global.cg.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(o.x), "f"(o.y), "f"(o.z), "f"(o.w) : "memory");
  } else {
    __stcs(p, o);
  }
#elif LP_STENCIL_ST == 1
  *p = o;  // plain (write-back)
#elif LP_STENCIL_ST == 2
  asm volatile("st.global.cg.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(o.x), "f"(o.y), "f"(o.z), "f"(o.w) : "memory");
#elif LP_STENCIL_ST == 3
  asm volatile("st.global.L1::no_allocate.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(o.x), "f"(o.y), "f"(o.z), "f"(o.w)
               : "memory");
#else
  __stcs(p, o);
#endif
}

__device__ __forceinline__ float4 ldg_nc_v4(const float* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
#ifndef LP_STENCIL_EDGE_LD
#define LP_STENCIL_EDGE_LD 0
#endif
__device__ __forceinline__ float ldg_nc_f(const float* p) {
  float r;
#if LP_STENCIL_EDGE_LD == 1
  asm volatile("ld.global.nc.L2::64B.f32 %0, [%1];" : "=f"(r) : "l"(p));
#elif LP_STENCIL_EDGE_LD == 2
  asm volatile("ld.global.f32 %0, [%1];" : "=f"(r) : "l"(p));
#elif LP_STENCIL_EDGE_LD == 3
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(p));
#else
  asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(r) : "l"(p));
#endif
  return r;
}

template <uint32_t MASK, int STORE, int COMBINE, int RWS = 16, int EL = 0>
__global__ void __launch_bounds__(kRM / RWS * 32, 2) stencil5_ldg_kernel(const float* __restrict__ in, int64_t ldi,
                                                              float* __restrict__ out, int64_t ldo, int row_lo,
                                                              int row_span, int W,
                                                              int64_t Q, int64_t R, uint32_t* __restrict__ ck,
                                                              int64_t rid_offset, const int64_t* __restrict__ list,
                                                              const int64_t* __restrict__ d_n) {
  constexpr int kRowsW = RWS, kNW = kRM / RWS, kNT = kNW * 32;  // rows per warp, warps, threads
  __shared__ CkRecord warp_rec[kNW];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  __shared__ int s_bad;
  const int64_t ntiles = (list && COMBINE != 2) ? *d_n : R;
  for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const int64_t rid = (list && COMBINE != 2) ? (list[t] - rid_offset) : t;
    const int64_t p = rid / Q, q = rid - p * Q;
    const int i0 = (int)(p * kRM) + wid * kRowsW;
    const int j = (int)(q * kRN) + lane * 4;
    if constexpr (COMBINE == 2) {
      // Listing 7 (L565-578): check-and-recover in the same grid as the original kernel --
      // validate this region from memory (L183), re-execute it only if the check fails.
      CkPartial<MASK> vp;
      AdlerRows vad;
#pragma unroll
      for (int r = 0; r < kRowsW; ++r) {
        const uint4 w4 = ld_stream_u4(out + (int64_t)(i0 + r) * ldo + j);
        add4_modxor(vp, w4.x, w4.y, w4.z, w4.w);
        if constexpr ((MASK & kAdler) != 0) vad.add_row(w4.x, w4.y, w4.z, w4.w);
      }
      if constexpr ((MASK & kAdler) != 0)
        vad.fold(vp, (uint32_t)(wid * kRowsW * kRN * 4 + lane * 16 + 1), kRowsW, kRN * 4);
      const CkRecord vr = warp_reduce<MASK>(vp);
      if (lane == 0) warp_rec[wid] = vr;
      __syncthreads();
      if (threadIdx.x == 0) {
        CkRecord rr = warp_rec[0];
#pragma unroll
        for (int w = 1; w < kNW; ++w) rr = combine(rr, warp_rec[w]);
        uint32_t words[3];
        record_words<MASK>(rr, (uint64_t)kRM * kRN * 4, words);
        constexpr int S = selem_of(MASK);
        bool bad = false;
        if constexpr (STORE == 0) {
#pragma unroll
          for (int s2 = 0; s2 < S; ++s2) bad |= (ck[rid * S + s2] != words[s2]);
        } else {
          uint32_t stored[3];
          bad = !store_lookup<S, STORE>(ck, (uint32_t)(rid + rid_offset), stored);
#pragma unroll
          for (int s2 = 0; s2 < S; ++s2) bad |= (!bad && stored[s2] != words[s2]);
        }
        s_bad = bad ? 1 : 0;
        if (bad) atomicAdd(reinterpret_cast<unsigned long long*>(const_cast<int64_t*>(d_n)), 1ull);
      }
      __syncthreads();
      if (!s_bad) continue;  // uniform across the CTA
    }
    const int je = lane == 0 ? j - 1 : j + 4;
    const bool eok = (lane == 0 || lane == 31) && je >= 0 && je < W;
    float4 v[kRowsW + 2];
    constexpr bool kEdgeLanes = (EL & 1) != 0, kTwoPhase = (EL & 2) != 0;
    float edge[kEdgeLanes ? 1 : kRowsW];
#pragma unroll
    for (int r = 0; r < kRowsW + 2; ++r) {
      const int i = i0 - 1 + r;
      v[r] = ((unsigned)(i - row_lo) < (unsigned)row_span) ? ldg_nc_v4(in + (int64_t)i * ldi + j) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    if constexpr (kEdgeLanes) {
      // edge columns by lane: lanes 0..RWS-1 hold the left edge (column q*128-1) of rows 0..RWS-1, lanes
      // RWS..2*RWS-1 the right edge (column q*128+128); broadcast to lanes 0 / 31 by shuffle per row
      const int jq = (int)(q * kRN), er = lane % kRowsW;
      const int jc = lane < kRowsW ? jq - 1 : jq + kRN;
      edge[0] = (lane < 2 * kRowsW && jc >= 0 && jc < W) ? ldg_nc_f(in + (int64_t)(i0 + er) * ldi + jc) : 0.f;
    } else {
#pragma unroll
      for (int r = 0; r < kRowsW; ++r) edge[r] = eok ? ldg_nc_f(in + (int64_t)(i0 + r) * ldi + je) : 0.f;
    }
    CkPartial<MASK> part;
    AdlerRows ad;
#pragma unroll
    for (int r = 0; r < kRowsW; ++r) {
      const float4 u = v[r], c = v[r + 1], d = v[r + 2];
      float left = __shfl_up_sync(0xFFFFFFFFu, c.w, 1);
      float right = __shfl_down_sync(0xFFFFFFFFu, c.x, 1);
      if constexpr (kEdgeLanes) {
        const float el = __shfl_sync(0xFFFFFFFFu, edge[0], r), er = __shfl_sync(0xFFFFFFFFu, edge[0], kRowsW + r);
        if (lane == 0) left = el;
        if (lane == 31) right = er;
      } else {
        if (lane == 0) left = edge[r];
        if (lane == 31) right = edge[r];
      }
      float4 o;
      o.x = st5(c.x, u.x, d.x, left, c.y);
      o.y = st5(c.y, u.y, d.y, c.x, c.z);
      o.z = st5(c.z, u.z, d.z, c.y, c.w);
      o.w = st5(c.w, u.w, d.w, c.z, right);
      st_out<kTwoPhase && (MASK & kAdler) != 0>(reinterpret_cast<float4*>(out + (int64_t)(i0 + r) * ldo + j), o);
      if constexpr (kTwoPhase) {
        v[r] = o;  // row r's input is dead: keep the stored vector for the checksum pass below
      } else if constexpr (MASK != 0) {
        add4_modxor(part, __float_as_uint(o.x), __float_as_uint(o.y), __float_as_uint(o.z), __float_as_uint(o.w));
        if constexpr ((MASK & kAdler) != 0)
          ad.add_row(__float_as_uint(o.x), __float_as_uint(o.y), __float_as_uint(o.z), __float_as_uint(o.w));
      }
    }
    if constexpr (kTwoPhase && MASK != 0) {
      // two-phase form: every row's store is issued before the checksum arithmetic starts (the warp
      // barrier keeps ptxas from hoisting the dp4a chains above the stores)
      __syncwarp();
      // Adler with four independent accumulator sets (rows r mod 4) so the dp4a chains overlap; the row
      // moment is summed directly (R = sum_r r * bs_r = n * S - T of AdlerRows): the same integer sums
      uint32_t aS[4] = {0, 0, 0, 0}, aR[4] = {0, 0, 0, 0}, aW[4] = {0, 0, 0, 0};
#pragma unroll
      for (int r = 0; r < kRowsW; ++r) {
        const float4 o = v[r];
        const uint32_t x = __float_as_uint(o.x), y = __float_as_uint(o.y), z = __float_as_uint(o.z),
                       w = __float_as_uint(o.w);
        add4_modxor(part, x, y, z, w);
        if constexpr ((MASK & kAdler) != 0) {
          const uint32_t bs = (uint32_t)__dp4a(x, 0x01010101u, __dp4a(y, 0x01010101u, 0u)) +
                              (uint32_t)__dp4a(z, 0x01010101u, __dp4a(w, 0x01010101u, 0u));
          aS[r & 3] += bs;
          aR[r & 3] += (uint32_t)r * bs;
          aW[r & 3] = (uint32_t)__dp4a(x, 0x03020100u, __dp4a(y, 0x07060504u,
                                       __dp4a(z, 0x0B0A0908u, __dp4a(w, 0x0F0E0D0Cu, aW[r & 3]))));
        }
      }
      if constexpr ((MASK & kAdler) != 0) {
        const uint32_t S = (aS[0] + aS[1]) + (aS[2] + aS[3]), Rm = (aR[0] + aR[1]) + (aR[2] + aR[3]),
                       Wl = (aW[0] + aW[1]) + (aW[2] + aW[3]);
        part.s += S;
        part.w += (uint64_t)(uint32_t)(wid * kRowsW * kRN * 4 + lane * 16 + 1) * S + (uint64_t)(kRN * 4) * Rm + Wl;
      }
    }
    if constexpr ((MASK & kAdler) != 0 && !kTwoPhase)
      ad.fold(part, (uint32_t)(wid * kRowsW * kRN * 4 + lane * 16 + 1), kRowsW, kRN * 4);
    if constexpr (MASK != 0 && COMBINE == 1) {
      // split-barrier combine (one region per CTA): every warp parks its partial in shared memory and
      // ARRIVES on named barrier 2 without waiting; only warp 0 waits (bar.sync) and then combines the
      // 8 partials (Listing 3) and stores the record.  No shared state needs initialising, and 7 of the
      // 8 warps retire as soon as their stores are issued.
      const CkRecord wr = warp_reduce<MASK>(part);
      if (lane == 0) warp_rec[wid] = wr;
      if (wid != 0) {
        asm volatile("bar.arrive 2, %0;" ::"n"(kNT) : "memory");
      } else {
        asm volatile("bar.sync 2, %0;" ::"n"(kNT) : "memory");
        if (lane == 0) {
          CkRecord rr = warp_rec[0];
#pragma unroll
          for (int w = 1; w < kNW; ++w) rr = combine(rr, warp_rec[w]);
          uint32_t words[3];
          record_words<MASK>(rr, (uint64_t)kRM * kRN * 4, words);
          store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
        }
      }
    } else if constexpr (MASK == 0 && COMBINE == 1 && LP_STENCIL_TWIN_BAR) {
      // the unprotected twin keeps the same split barrier, so the LP overhead compares like with like
      if (wid != 0) asm volatile("bar.arrive 2, %0;" ::"n"(kNT) : "memory");
      else asm volatile("bar.sync 2, %0;" ::"n"(kNT) : "memory");
    } else if constexpr (MASK != 0) {
      const CkRecord wr = warp_reduce<MASK>(part);
      __syncthreads();  // warp_rec may still be read by the check phase (COMBINE == 2)
      if (lane == 0) warp_rec[wid] = wr;
      __syncthreads();
      if (threadIdx.x == 0) {
        CkRecord rr = warp_rec[0];
#pragma unroll
        for (int w = 1; w < kNW; ++w) rr = combine(rr, warp_rec[w]);
        uint32_t words[3];
        record_words<MASK>(rr, (uint64_t)kRM * kRN * 4, words);
        store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
      }
      if (list || COMBINE == 2) __syncthreads();
    }
  }
}


// ---- TMA-fed persistent form of the full run (one CTA per SM; A/B, LP_STENCIL_TMA=1, not the default) ----
//
// Per region, three cp.async.bulk.tensor boxes land in one stage of a 3-deep ring: the 130 x 128 centre
// (region rows -1 .. 128, line-aligned) and the 4-column halo strips left and right.  The tensor maps
// cover only this shard's readable rows [row_lo, row_lo + row_span) and the W domain columns, so TMA's
// out-of-bounds zero fill IS the stencil's zero boundary (R19).  Warp NW (one lane) is the producer and
// keeps two regions in flight ahead of the consumers, whatever the consumers' checksum epilogue costs;
// it also combines the NW warp partials (Listing 3) and stores the record (L349) once a stage is
// released.  Consumer warps read the stage from shared memory (one 16-B vector per row, conflict-free)
// with the same lane -> column mapping and per-lane partials as the LDG form.
// Measured (profiles/r02/ab_stencil_tma.txt): Adler costs only +1.6% over THIS form's twin, but the twin
// itself takes 1.57-1.70 ms against the LDG form's 1.29 ms: with the output stores in the mix the halo
// strips are re-read from DRAM (5.14 vs 4.35 GB read), and even without halos (diagnostic build) TMA +
// stores ran 1.43 ms.  So the LDG form stays the default and Adler's +8% stands against it.
constexpr int kTmaBoxR = kRM + 2;                                  // region rows -1 .. 128
constexpr int kTmaHaloL = kTmaBoxR * kRN * 4;                          // 66 560: centre box [130][128]
constexpr int kTmaHaloR = kTmaHaloL + ((kTmaBoxR * 16 + 127) / 128) * 128;  // left halo [130][4] (cols -4..-1)
constexpr int kTmaStageBytes = ((kTmaHaloR + kTmaBoxR * 16 + 127) / 128) * 128;  // right halo [130][4] (128..131)
constexpr uint32_t kTmaStageTx = kTmaBoxR * (kRN + 8) * 4;                // 70 720 B per region

__host__ __device__ constexpr int stencil_tma_smem(int stages) {
  return stages * kTmaStageBytes + stages * (2 * 8 + 16 * (int)sizeof(CkRecord) + 8) + 128;
}

__device__ __forceinline__ float4 lds_v4(uint32_t a) {
  float4 r;
  asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "r"(a));
  return r;
}
__device__ __forceinline__ float lds_f(uint32_t a) {
  float r;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(r) : "r"(a));
  return r;
}

template <uint32_t MASK, int STORE, int NW>
__global__ void __launch_bounds__((NW + 1) * 32, 1)
    stencil5_tma_kernel(const __grid_constant__ CUtensorMap tctr, const __grid_constant__ CUtensorMap thalo,
                        float* __restrict__ out, int64_t ldo, int row_lo, int64_t Q, int64_t R,
                        uint32_t* __restrict__ ck, int64_t rid_offset, int stages,
                        const int64_t* __restrict__ list, const int64_t* __restrict__ d_n) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + stages * kTmaStageBytes);
  uint64_t* empty = full + stages;
  CkRecord* srec = reinterpret_cast<CkRecord*>(empty + stages);  // [stages][NW]
  constexpr int RW = kRM / NW;  // region rows per consumer warp
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t first = blockIdx.x, stride = gridDim.x;
  const int64_t nwork = list ? *d_n : R;  // list mode (recovery): the failed list's entries
  const int64_t niter = first < nwork ? (nwork - 1 - first) / stride + 1 : 0;
  int64_t* s_rid = reinterpret_cast<int64_t*>(smem_raw + stencil_tma_smem(stages) - 128 - stages * 8);
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], NW);
    }
    fence_barrier_init();
  }
  __syncthreads();

  if (wid == NW) {  // producer (+ record store)
    if (lane != 0) return;
    prefetch_tmap(&tctr);
    prefetch_tmap(&thalo);
    auto finish = [&](int64_t it, int s) {
      if constexpr (MASK != 0) {
        const int64_t rid = s_rid[s];
        CkRecord rr = srec[s * NW];
#pragma unroll
        for (int w = 1; w < NW; ++w) rr = combine(rr, srec[s * NW + w]);
        uint32_t words[3];
        record_words<MASK>(rr, (uint64_t)kRM * kRN * 4, words);
        store_record<MASK, STORE>(ck, rid, (uint32_t)(rid + rid_offset), words);
      }
    };
    for (int64_t it = 0; it < niter; ++it) {
      const int s = (int)(it % stages);
      const uint32_t k = (uint32_t)(it / stages);
      if (it >= stages) {
        mbar_wait(&empty[s], (k & 1u) ^ 1u);  // the stage's previous region (it - stages) is consumed
        finish(it - stages, s);
      }
      const int64_t rid = list ? list[first + it * stride] - rid_offset : first + it * stride;
      const int64_t p = rid / Q, q = rid - p * Q;
      s_rid[s] = rid;  // published to the consumers by the full barrier's completion
      mbar_expect_tx(&full[s], kTmaStageTx);
      const int c0 = (int)(q * kRN), r0 = (int)(p * kRM) - 1 - row_lo;
      uint8_t* dst = smem_raw + s * kTmaStageBytes;
      // the 128 region columns as one line-aligned box, the 4-column halo strips left and right apart
      tma_load_2d(&tctr, &full[s], dst, c0, r0);
      tma_load_2d(&thalo, &full[s], dst + kTmaHaloL, c0 - 4, r0);
      tma_load_2d(&thalo, &full[s], dst + kTmaHaloR, c0 + kRN, r0);
    }
    for (int64_t it = niter > stages ? niter - stages : 0; it < niter; ++it) {
      const int s = (int)(it % stages);
      mbar_wait(&empty[s], (uint32_t)(it / stages) & 1u);
      finish(it, s);
    }
    return;
  }

  // consumers: warp wid owns region rows wid*RW .. wid*RW+RW-1 (box rows +1), lane owns columns lane*4 .. +3
  const uint32_t sbase = smem_u32(smem_raw);
  const uint32_t lane_off = (uint32_t)((wid * RW) * kRN * 4 + lane * 16);
  const uint32_t edge_off = (uint32_t)((lane < 16 ? kTmaHaloL + 12 : kTmaHaloR) + (wid * RW + 1) * 16);
  for (int64_t it = 0; it < niter; ++it) {
    const int s = (int)(it % stages);
    mbar_wait(&full[s], (uint32_t)(it / stages) & 1u);
    const int64_t rid = s_rid[s], p = rid / Q, q = rid - p * Q;
    const uint32_t st0 = sbase + (uint32_t)s * kTmaStageBytes;
    float* orow = out + (p * kRM + wid * RW) * ldo + q * kRN + lane * 4;
    float4 u = lds_v4(st0 + lane_off), c = lds_v4(st0 + lane_off + kRN * 4);
    CkPartial<MASK> part;
    AdlerRows ad;
#pragma unroll
    for (int r = 0; r < RW; ++r) {
      const float4 d = lds_v4(st0 + lane_off + (r + 2) * kRN * 4);
      const float e = lds_f(st0 + edge_off + r * 16);
      float left = __shfl_up_sync(0xFFFFFFFFu, c.w, 1);
      float right = __shfl_down_sync(0xFFFFFFFFu, c.x, 1);
      if (lane == 0) left = e;
      if (lane == 31) right = e;
      float4 o;
      o.x = st5(c.x, u.x, d.x, left, c.y);
      o.y = st5(c.y, u.y, d.y, c.x, c.z);
      o.z = st5(c.z, u.z, d.z, c.y, c.w);
      o.w = st5(c.w, u.w, d.w, c.z, right);
#if LP_STENCIL_TMA_ST_CG
      st_out<true>(reinterpret_cast<float4*>(orow + (int64_t)r * ldo), o);
#else
      __stcs(reinterpret_cast<float4*>(orow + (int64_t)r * ldo), o);
#endif
      if constexpr (MASK != 0) {
        add4_modxor(part, __float_as_uint(o.x), __float_as_uint(o.y), __float_as_uint(o.z), __float_as_uint(o.w));
        if constexpr ((MASK & kAdler) != 0)
          ad.add_row(__float_as_uint(o.x), __float_as_uint(o.y), __float_as_uint(o.z), __float_as_uint(o.w));
      }
      u = c;
      c = d;
    }
    if constexpr (MASK != 0) {
      if constexpr ((MASK & kAdler) != 0) ad.fold(part, (uint32_t)(wid * RW * kRN * 4 + lane * 16 + 1), RW, kRN * 4);
      const CkRecord wr = warp_reduce<MASK>(part);
      if (lane == 0) srec[s * NW + wid] = wr;
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);
  }
}

int stencil_tma_stages() {
  static int v = [] {
    const char* e = getenv("LP_STENCIL_STAGES");
    const int s = e ? atoi(e) : 3;
    return s < 2 ? 2 : (s > 3 ? 3 : s);
  }();
  return v;
}
CUtensorMapL2promotion stencil_tma_promo() {
  static CUtensorMapL2promotion v = [] {
    const char* e = getenv("LP_STENCIL_PROMO");
    const int b = e ? atoi(e) : 64;
    return b == 256 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B
                    : (b == 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
                                : (b == 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B : CU_TENSOR_MAP_L2_PROMOTION_NONE));
  }();
  return v;
}
int stencil_tma_warps() {
  static int v = [] {
    const char* e = getenv("LP_STENCIL_NW");
    return (e && atoi(e) == 8) ? 8 : 16;
  }();
  return v;
}
// full run, LDG form, bit 0: edge columns loaded by lanes and broadcast by shuffle (one register instead
// of 16), bit 1: two-phase epilogue (every row stored before the checksum pass).  Default: both for the
// protected kernels (frees the registers the Adler accumulators need and keeps ptxas from scheduling the
// dp4a chains ahead of the stores: Adler +7% -> +1%, profiles/r02/ab_stencil_epilogue.txt), neither for
// the unprotected twin (its fastest form, so the LP overhead is measured against the fastest plain kernel).
int stencil_edge_lanes(uint32_t mask) {
  static int v = [] {
    const char* e = getenv("LP_STENCIL_EL");
    return e ? (atoi(e) == 3 ? 3 : 0) : -1;  // A/B override: 0 or 3 for every kernel
  }();
  return v >= 0 ? v : (mask ? 3 : 0);
}
// list-mode recovery through the TMA-fed form (default): the producer reads the failed list ahead and keeps
// two scattered regions in flight per SM; the LDG form re-executes them one region per CTA at a time
// (232 -> 185 us for 10% of C4, profiles/r02/ab_stencil_tma.txt)
bool stencil_tma_list() {
  static bool v = [] {
    const char* e = getenv("LP_STENCIL_TMA_LIST");
    return e ? atoi(e) != 0 : true;
  }();
  return v;
}
bool stencil_use_tma() {
  static bool v = [] {
    const char* e = getenv("LP_STENCIL_TMA");
    return e ? atoi(e) != 0 : false;
  }();
  return v;
}

cudaError_t launch_stencil_tma(const StencilArgs& a, int64_t Q, int64_t R, cudaStream_t st) {
  CUtensorMap tm, tt;
  const int nw = stencil_tma_warps();
  // rows [row_lo, row_lo + row_span) of the shard, columns [0, W): everything else reads as zero
  const float* base = a.in + (int64_t)a.row_lo * a.ldi;
  const CUtensorMapL2promotion promo = stencil_tma_promo();
  if (!tma_map_2d(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, base, (uint64_t)a.W, (uint64_t)a.row_span,
                  (uint64_t)a.ldi, kRN, kTmaBoxR, CU_TENSOR_MAP_SWIZZLE_NONE, promo) ||
      !tma_map_2d(&tt, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, base, (uint64_t)a.W, (uint64_t)a.row_span,
                  (uint64_t)a.ldi, 4, kTmaBoxR, CU_TENSOR_MAP_SWIZZLE_NONE, promo))
    return cudaErrorInvalidValue;
  const int stages = stencil_tma_stages();
  const int smem = stencil_tma_smem(stages);
  int64_t grid = (a.list || R >= a.sm_count) ? a.sm_count : R;
  if (grid < 1) grid = 1;
  const int sk = a.mask ? a.hash.store : 0;
  cudaError_t e = cudaSuccess;
  switch (a.mask * 5 + sk) {
#define LP_TCASE(M, S)                                                                                       \
  case M * 5 + S: {                                                                                          \
    auto kfn = nw == 16 ? stencil5_tma_kernel<M, S, 16> : stencil5_tma_kernel<M, S, 8>;                      \
    e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);                        \
    if (e != cudaSuccess) return e;                                                                          \
    kfn<<<(unsigned)grid, (nw + 1) * 32, smem, st>>>(tm, tt, a.out, a.ldo, a.row_lo, Q, R, a.ck, a.rid_offset, \
                                                     stages, a.list, a.d_n);                                 \
    break;                                                                                                   \
  }
#define LP_TCASE3(M) LP_TCASE(M, 0)
#define LP_TCASE5(M) LP_TCASE(M, 0) LP_TCASE(M, 1) LP_TCASE(M, 2) LP_TCASE(M, 3) LP_TCASE(M, 4)
    LP_TCASE(0, 0)
    LP_TCASE5(1)
    LP_TCASE3(2)
    LP_TCASE5(3)
    LP_TCASE3(4)
    LP_TCASE3(5)
    LP_TCASE3(6)
    LP_TCASE3(7)
#undef LP_TCASE3
#undef LP_TCASE5
#undef LP_TCASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace

bool stencil_supported(int RM, int RN) { return RM == kRM && RN == kRN; }

cudaError_t launch_stencil(const StencilArgs& a, cudaStream_t st) {
  const int64_t Q = a.W / kRN, R = (a.H / kRM) * Q;
  if (a.H > (int64_t)INT32_MAX / 2 || a.W > (int64_t)INT32_MAX / 2) return cudaErrorInvalidValue;
  if (a.list ? stencil_tma_list() : stencil_use_tma()) return launch_stencil_tma(a, Q, R, st);
  const int sk = a.mask ? a.hash.store : 0;
  // full run: one region per CTA, barrier-free combine; list mode (recovery):
  // persistent CTAs over the failed list, barrier combine (accumulators reused)
  // list mode: 2 persistent CTAs per SM (the occupancy limit); 8 / 32 / 64 per SM, and one region per CTA over
  // R CTAs with the split-barrier combine, measured the same recovery phase
  int64_t grid = a.list ? (R < a.sm_count * 2 ? R : a.sm_count * 2) : R;
  if (grid < 1) grid = 1;
  switch (a.mask * 5 + sk) {
#define LP_LCASE(M, S)                                                                                          \
  case M * 5 + S:                                                                                               \
    if (a.list)                                                                                                 \
      stencil5_ldg_kernel<M, S, 0><<<(unsigned)grid, 256, 0, st>>>(a.in, a.ldi, a.out, a.ldo, a.row_lo,          \
                                                                   a.row_span, (int)a.W, Q, R, a.ck, a.rid_offset, a.list,   \
                                                                   a.d_n);                                      \
    else if (stencil_edge_lanes(a.mask) == 3)                                                                   \
      stencil5_ldg_kernel<M, S, 1, 16, 3><<<(unsigned)grid, 256, 0, st>>>(a.in, a.ldi, a.out, a.ldo, a.row_lo,   \
                                                                   a.row_span, (int)a.W, Q, R, a.ck, a.rid_offset, a.list,   \
                                                                   a.d_n);                                      \
    else                                                                                                        \
      stencil5_ldg_kernel<M, S, 1><<<(unsigned)grid, 256, 0, st>>>(a.in, a.ldi, a.out, a.ldo, a.row_lo,          \
                                                                   a.row_span, (int)a.W, Q, R, a.ck, a.rid_offset, a.list,   \
                                                                   a.d_n);                                      \
    break;
#define LP_LCASE3(M) LP_LCASE(M, 0)
#define LP_LCASE5(M) LP_LCASE(M, 0) LP_LCASE(M, 1) LP_LCASE(M, 2) LP_LCASE(M, 3) LP_LCASE(M, 4)
    LP_LCASE(0, 0)
    LP_LCASE5(1)
    LP_LCASE3(2)
    LP_LCASE5(3)
    LP_LCASE3(4)
    LP_LCASE3(5)
    LP_LCASE3(6)
    LP_LCASE3(7)
#undef LP_LCASE3
#undef LP_LCASE5
#undef LP_LCASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_stencil_check_recover(const StencilArgs& a, int64_t* d_recovered, cudaStream_t st) {
  const int64_t Q = a.W / kRN, R = (a.H / kRM) * Q;
  if (a.H > (int64_t)INT32_MAX / 2 || a.W > (int64_t)INT32_MAX / 2 || a.mask == 0) return cudaErrorInvalidValue;
  cudaError_t e = cudaMemsetAsync(d_recovered, 0, sizeof(int64_t), st);
  if (e != cudaSuccess) return e;
  const int sk = a.hash.store;
  switch (a.mask * 5 + sk) {
#define LP_CCASE(M, S)                                                                                          \
  case M * 5 + S:                                                                                               \
    stencil5_ldg_kernel<M, S, 2, 16, 3><<<(unsigned)R, 256, 0, st>>>(a.in, a.ldi, a.out, a.ldo, a.row_lo, a.row_span,  \
                                                              (int)a.W, Q,                                      \
                                                              R, a.ck, a.rid_offset, nullptr, d_recovered);     \
    break;
#define LP_CCASE3(M) LP_CCASE(M, 0)
#define LP_CCASE5(M) LP_CCASE(M, 0) LP_CCASE(M, 1) LP_CCASE(M, 2) LP_CCASE(M, 3) LP_CCASE(M, 4)
    LP_CCASE5(1)
    LP_CCASE3(2)
    LP_CCASE5(3)
    LP_CCASE3(4)
    LP_CCASE3(5)
    LP_CCASE3(6)
    LP_CCASE3(7)
#undef LP_CCASE3
#undef LP_CCASE5
#undef LP_CCASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace lp
