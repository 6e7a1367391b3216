// lp_kernels.cu -- validation, compaction, table init, crash injection, stats.
//
// Validation is the recovery kernel's first half (L183 §IV-A): "fetching the
// corresponding data from memory, computing their checksums, and then
// comparing them with the ones stored in the checksum table".  On B200 it is an
// HBM-streaming reduction: one warp per region, 16-byte non-allocating loads,
// eight loads in flight per lane, one redux.sync per checksum.  The failed
// regions are then compacted into an ascending list (Reading R12/R13) so that
// recovery re-executes only those.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>
#include <stdlib.h>

#include "lp_device.cuh"
#include "lp_internal.h"

namespace lp {
namespace {

constexpr int kValThreads = 256;
constexpr int kValWarps = kValThreads / 32;
constexpr int64_t kMaxValCtas = 148 * 16 * 4;
constexpr int kValUnroll = 8;
// CTAs per SM the validate kernel is compiled for when Adler is in the record: 4 (64 registers) spills ~100 B
// per thread with the Adler accumulators; 3 gives them 80 registers (A/B: profiles/r02/ab_validate_adler.txt)
#ifndef LP_VAL_ADLER_MINB
#define LP_VAL_ADLER_MINB 3
#endif

// Segmented reduction of the per-lane partials over aligned groups of 2^lg_log2
// lanes (one group = one region).  A whole-warp group uses one redux.sync per
// checksum (the B200 form of Listing 4's shfl_down ladder, L244-258); narrower
// groups use an xor butterfly of log2(group) shuffles.  Adler's W is reduced
// mod 65521 per lane first so the u32 sums cannot wrap (<= 32 * 65520).


// Fused ordered compaction (a9) for small tables: every validate CTA bumps a ticket after
// its flags and count are written; the last one to arrive (it sees ticket == grid - 1)
// turns flags[0, R) into the ascending list of failed global rids + the device count, and
// resets the ticket for the next call.  Ordering: bar.sync, then a gpu-scope fence and the
// ticket RMW by thread 0 (cumulative: the CTA's flag stores are visible before the
// ticket moves); the last CTA fences again before reading the flags (L2: ld.global.cg).
__device__ __forceinline__ void fused_compact_if_last(const uint8_t* flags, int64_t R, int64_t rid_offset,
                                                      uint32_t* ticket, int64_t* list, int64_t* d_n,
                                                      NvlsCount nvc) {
  __shared__ int s_last;
  __shared__ int s_warp[kValWarps];
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  // thread t owns the 16-byte-aligned flag range [t * per, (t + 1) * per), per = 16 * nv <= 64:
  // nv independent 16-B loads (flags are 0/1 bytes, so popc of a word counts its set flags)
  constexpr int kMaxV = (int)(kFusedCompactMaxR / kValThreads / 16);
  const int nv = (int)((R + kValThreads * 16 - 1) / (kValThreads * 16));
  const int64_t i0 = (int64_t)threadIdx.x * nv * 16;
  uint4 fv[kMaxV];
  int c = 0;
#pragma unroll
  for (int u = 0; u < kMaxV; ++u) {
    fv[u] = make_uint4(0u, 0u, 0u, 0u);
    const int64_t b = i0 + u * 16;
    if (u < nv && b < R) {
      if (b + 16 <= R) {
        fv[u] = __ldcg(reinterpret_cast<const uint4*>(flags + b));
      } else {  // the table's ragged end
        uint32_t w[4] = {0u, 0u, 0u, 0u};
        for (int k = 0; k < (int)(R - b); ++k) w[k >> 2] |= (uint32_t)__ldcg(flags + b + k) << (8 * (k & 3));
        fv[u] = make_uint4(w[0], w[1], w[2], w[3]);
      }
    }
    c += __popc(fv[u].x) + __popc(fv[u].y) + __popc(fv[u].z) + __popc(fv[u].w);
  }
  // block exclusive scan of c
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int x = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xFFFFFFFFu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[wid] = x;
  __syncthreads();
  int woff = 0, total = 0;
#pragma unroll
  for (int w = 0; w < kValWarps; ++w) {
    const int v = s_warp[w];
    if (w < wid) woff += v;
    total += v;
  }
  int64_t pos = woff + x - c;
  if (c > 0) {
#pragma unroll
    for (int u = 0; u < kMaxV; ++u) {
      const uint32_t w4[4] = {fv[u].x, fv[u].y, fv[u].z, fv[u].w};
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint32_t m = w4[q];
        while (m) {  // set bytes in ascending order
          const int bit = __ffs(m) - 1;
          list[pos++] = rid_offset + i0 + u * 16 + q * 4 + (bit >> 3);
          m &= m - 1;
        }
      }
    }
  }
  if (threadIdx.x == 0) {
    *d_n = total;
    *ticket = 0u;
    nvls_publish(nvc, total);
  }
}

// Validate (a8): a warp task is a strip of G = 2^g_log2 horizontally adjacent
// regions (consecutive rids), LG = 32 / G lanes per region.  Lane li of a group
// reads the 16-byte chunks li, li + LG, ... of its region in row-major order, so
// the group's lanes cover LG / cpr whole region rows per load instruction (or
// 1 / (cpr / LG) of a row) and the warp touches G adjacent row segments.  Eight
// 16-byte non-allocating loads are in flight per lane.  G is chosen on the host
// (plan_validate) so that enough warps exist to keep ~16 MiB of reads in flight
// (1 region per warp for 128x128) while strips of small regions still give
// 256-512 B contiguous segments.  Each CTA owns a contiguous range of regions and
// writes its failure count for the ordered compaction.
// MODE 0 = compare with array table, 1 = compare with a quad hash table (lookup
// by global rid), 2 = write records (no compare), 3 = compare with a cuckoo table,
// 4 = count-only re-validation of the regions NOT flagged by the previous validate
// (flags read as the skip mask, mismatches added to *(u64*)d_n; array table) --
// runs beside the recovery of the flagged ones (lp_recover_revalidate).
template <uint32_t MASK, int MODE, int MB = 4>
__global__ void __launch_bounds__(kValThreads, MB) validate_kernel(const uint8_t* __restrict__ out, int64_t ldc_bytes,
                                                                int64_t Q, int64_t R, int RM, int row_bytes,
                                                                int cpr_log2, int g_log2,
                                                                const uint32_t* __restrict__ ck,
                                                                int64_t rid_offset, uint8_t* __restrict__ flags,
                                                                uint32_t* __restrict__ records, int64_t rpc,
                                                                uint32_t* __restrict__ cta_counts,
                                                                uint32_t* __restrict__ ticket,
                                                                int64_t* __restrict__ list, int64_t* __restrict__ d_n,
                                                                NvlsCount nv) {
  constexpr int S = selem_of(MASK);
  __shared__ uint32_t s_fail;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int lg_log2 = 5 - g_log2;                       // lanes per region (log2)
  const int G = 1 << g_log2;
  const int gi = lane >> lg_log2, li = lane & ((1 << lg_log2) - 1);
  const int chunks = RM << cpr_log2;                    // 16-byte chunks per region
  const int cmask = (1 << cpr_log2) - 1;
  const uint64_t nbytes = (uint64_t)RM * (uint64_t)row_bytes;
  // let the compaction grid (programmatic dependent launch) be scheduled early; it
  // waits in griddepcontrol.wait until this whole grid has completed and flushed
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x == 0) s_fail = 0;
  __syncthreads();
  const int64_t r0 = (int64_t)blockIdx.x * rpc;
  const int64_t r1 = r0 + rpc < R ? r0 + rpc : R;
  for (int64_t t0 = r0 + (int64_t)warp * G; t0 < r1; t0 += (int64_t)kValWarps * G) {
    const int64_t r = t0 + gi;
    const bool live = r < r1 && (MODE != 4 || !flags[r]);
    const int64_t p = r / Q, q = r - p * Q;
    const uint8_t* base = out + p * (int64_t)RM * ldc_bytes + q * (int64_t)row_bytes;
    CkPartial<MASK> part;
    // Adler column form: when a lane's chunks all sit in one column of the region (LG >= cpr, the planned
    // geometries), chunk j of the lane is at byte position pos0 + j * dpos, so sum_j pos_j * bs_j =
    // pos0 * S + dpos * J with J = sum_j j * bs_j: no per-chunk position or 64-bit multiply, and the per-chunk
    // dp4a chains are independent (the 64-bit position chain of add4 is what held the next loads back)
    const bool colform = ((MASK & kAdler) != 0) && lg_log2 >= cpr_log2 && ((chunks >> lg_log2) <= 1024);
    uint32_t aS = 0, aJ = 0, aW = 0;
    for (int c0 = li, jb = 0; c0 < chunks; c0 += kValUnroll << lg_log2, jb += kValUnroll) {
      uint4 v[kValUnroll];
#pragma unroll
      for (int u = 0; u < kValUnroll; ++u) {
        const int c = c0 + (u << lg_log2);
        if (live && c < chunks) v[u] = ld_stream_u4(base + (int64_t)(c >> cpr_log2) * ldc_bytes + ((c & cmask) << 4));
      }
      if (colform) {
#pragma unroll
        for (int u = 0; u < kValUnroll; ++u) {
          const int c = c0 + (u << lg_log2);
          if (live && c < chunks) {
            if constexpr ((MASK & kMod) != 0) part.mod += (v[u].x + v[u].y) + (v[u].z + v[u].w);
            if constexpr ((MASK & kXor) != 0) part.xr ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
            const uint32_t bs = (uint32_t)__dp4a(v[u].x, 0x01010101u, __dp4a(v[u].y, 0x01010101u, 0u)) +
                                (uint32_t)__dp4a(v[u].z, 0x01010101u, __dp4a(v[u].w, 0x01010101u, 0u));
            const uint32_t ws = (uint32_t)__dp4a(v[u].x, 0x03020100u, __dp4a(v[u].y, 0x07060504u,
                                           __dp4a(v[u].z, 0x0B0A0908u, __dp4a(v[u].w, 0x0F0E0D0Cu, 0u))));
            aS += bs;
            aJ += (uint32_t)(jb + u) * bs;
            aW += ws;
          }
        }
      } else {
#pragma unroll
        for (int u = 0; u < kValUnroll; ++u) {
          const int c = c0 + (u << lg_log2);
          if (live && c < chunks) {
            const uint32_t pos = (uint32_t)((c >> cpr_log2) * row_bytes + ((c & cmask) << 4) + 1);
            part.add4(v[u].x, v[u].y, v[u].z, v[u].w, pos);
          }
        }
      }
    }
    if constexpr ((MASK & kAdler) != 0) {
      if (colform) {
        const uint32_t pos0 = (uint32_t)((li >> cpr_log2) * row_bytes + ((li & cmask) << 4) + 1);
        const uint32_t dpos = (uint32_t)((1 << (lg_log2 - cpr_log2)) * row_bytes);
        part.s += aS;
        part.w += (uint64_t)pos0 * aS + (uint64_t)dpos * aJ + aW;
      }
    }
    const CkRecord rec = segment_reduce<MASK>(part, lg_log2);
    if (live && li == 0) {
      uint32_t w[3];
      record_words<MASK>(rec, nbytes, w);
      if constexpr (MODE == 2) {
#pragma unroll
        for (int s = 0; s < S; ++s) records[r * S + s] = w[s];
      } else {
        bool bad = false;
        if constexpr (MODE == 0 || MODE == 4) {
#pragma unroll
          for (int s = 0; s < S; ++s) bad |= (ck[r * S + s] != w[s]);
        } else {
          uint32_t stored[3];
          bad = MODE == 3 ? !cuckoo_lookup<S>(ck, (uint32_t)(r + rid_offset), stored)
                          : !quad_lookup<S>(ck, (uint32_t)(r + rid_offset), stored);
#pragma unroll
          for (int s = 0; s < S; ++s) bad |= (!bad && stored[s] != w[s]);
        }
        if constexpr (MODE == 4) {
          if (bad) atomicAdd(reinterpret_cast<unsigned long long*>(d_n), 1ull);
        } else {
          flags[r] = bad ? 1 : 0;
          if (bad) atomicAdd(&s_fail, 1u);
        }
      }
    }
  }
  if constexpr (MODE != 2 && MODE != 4) {
    __syncthreads();
    if (threadIdx.x == 0) cta_counts[blockIdx.x] = s_fail;
    if (ticket) fused_compact_if_last(flags, R, rid_offset, ticket, list, d_n, nv);
  }
}

struct ValLaunch {
  dim3 grid;
  int64_t rpc;
  int g_log2;
};

template <uint32_t MASK>
cudaError_t validate_dispatch_mode(int mode, int mb, const ValLaunch& L, cudaStream_t st, const uint8_t* out,
                                   int64_t ldc_bytes, int64_t Q, int64_t R, int RM, int row_bytes, int cpr_log2,
                                   const uint32_t* ck, int64_t rid_offset, uint8_t* flags, uint32_t* records,
                                   uint32_t* counts, uint32_t* ticket, int64_t* list, int64_t* d_n,
                                   const NvlsCount& nv) {
#define LP_VLAUNCH1(MD, MB)                                                                               \
  validate_kernel<MASK, MD, MB><<<L.grid, kValThreads, 0, st>>>(out, ldc_bytes, Q, R, RM, row_bytes, cpr_log2,     \
                                                            L.g_log2, ck, rid_offset, flags, records, L.rpc, counts, \
                                                            ticket, list, d_n, nv)
#define LP_VLAUNCH(MD)                   \
  do {                                   \
    if (mb == LP_VAL_ADLER_MINB)         \
      LP_VLAUNCH1(MD, LP_VAL_ADLER_MINB); \
    else                                 \
      LP_VLAUNCH1(MD, 4);                \
  } while (0)
  if (mode == 0) LP_VLAUNCH(0);
  else if (mode == 4) LP_VLAUNCH(4);
  else if (mode == 1) LP_VLAUNCH(1);
  else if (mode == 3) LP_VLAUNCH(3);
  else LP_VLAUNCH(2);
#undef LP_VLAUNCH1
#undef LP_VLAUNCH
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Ordered compaction: flags[R] -> ascending list of global rids + count.
constexpr int kCompactThreads = 256;
constexpr int kCompactPerThread = 32;  // two uint4 of flags
constexpr int kCompactChunk = kCompactThreads * kCompactPerThread;

__device__ __forceinline__ int count_flags_u4(uint4 v) {
  // flags are 0/1 bytes
  return __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
}

__device__ __forceinline__ void load_flags(const uint8_t* flags, int64_t R, int64_t idx0, uint32_t f[8]) {
  if (idx0 + kCompactPerThread <= R && ((((uintptr_t)(flags + idx0)) & 15u) == 0)) {
    const uint4 a = *reinterpret_cast<const uint4*>(flags + idx0);
    const uint4 b = *reinterpret_cast<const uint4*>(flags + idx0 + 16);
    f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w;
    f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
  } else {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      uint32_t w = 0;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int64_t k = idx0 + i * 4 + j;
        if (k < R && flags[k]) w |= 1u << (8 * j);
      }
      f[i] = w;
    }
  }
}

__device__ __forceinline__ int block_exclusive_scan(int v, int* smem_warp, int* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xFFFFFFFFu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) smem_warp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    int s = lane < kCompactThreads / 32 ? smem_warp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xFFFFFFFFu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < kCompactThreads / 32) smem_warp[lane] = s;  // inclusive
  }
  __syncthreads();
  const int warp_off = wid ? smem_warp[wid - 1] : 0;
  *total = smem_warp[kCompactThreads / 32 - 1];
  return warp_off + x - v;
}

__global__ void __launch_bounds__(kCompactThreads) compact_count_kernel(const uint8_t* __restrict__ flags, int64_t R,
                                                                        uint32_t* __restrict__ block_counts) {
  __shared__ int warp_s[kCompactThreads / 32];
  const int64_t idx0 = (int64_t)blockIdx.x * kCompactChunk + (int64_t)threadIdx.x * kCompactPerThread;
  uint32_t f[8];
  load_flags(flags, R, idx0, f);
  int c = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) c += __popc(f[i]);
  int total;
  block_exclusive_scan(c, warp_s, &total);
  if (threadIdx.x == 0) block_counts[blockIdx.x] = (uint32_t)total;
}

__global__ void __launch_bounds__(kCompactThreads) compact_scatter_kernel(const uint8_t* __restrict__ flags, int64_t R,
                                                                          const uint32_t* __restrict__ block_counts,
                                                                          int nblocks, int64_t chunk, int per_block,
                                                                          int64_t rid_offset,
                                                                          int64_t* __restrict__ list,
                                                                          int64_t* __restrict__ d_n, NvlsCount nv) {
  // counting block i (i < nblocks) owns flags [i*chunk, (i+1)*chunk); this scatter block
  // owns counting blocks [b*per_block, (b+1)*per_block).  Its output offset is the sum of
  // the counts before its first counting block (block 0 also publishes the total).
  __shared__ int warp_s[kCompactThreads / 32];
  __shared__ long long red[2][kCompactThreads / 32];
  __shared__ long long s_base;
  // launched as a programmatic dependent of the validate grid: wait for its counts/flags
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const int first = (int)blockIdx.x * per_block;
  long long mine = 0, all = 0;
  for (int b = threadIdx.x; b < nblocks; b += kCompactThreads) {
    const long long c = block_counts[b];
    if (b < first) mine += c;
    if (blockIdx.x == 0) all += c;
    else if (b >= first) break;
  }
  for (int o = 16; o > 0; o >>= 1) {
    mine += __shfl_xor_sync(0xFFFFFFFFu, mine, o);
    all += __shfl_xor_sync(0xFFFFFFFFu, all, o);
  }
  if ((threadIdx.x & 31) == 0) {
    red[0][threadIdx.x >> 5] = mine;
    red[1][threadIdx.x >> 5] = all;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    long long m = 0, a = 0;
    for (int w = 0; w < kCompactThreads / 32; ++w) {
      m += red[0][w];
      a += red[1][w];
    }
    s_base = m;
    if (blockIdx.x == 0) {
      *d_n = a;
      nvls_publish(nv, a);
    }
  }
  __syncthreads();
  long long base = s_base;
  const int64_t lo = (int64_t)first * chunk;
  int64_t hi = (int64_t)(first + per_block) * chunk;
  if (hi > R) hi = R;
  // 16 flags per thread per pass (two 8-byte loads: lo is a multiple of 8 because every validate
  // CTA owns a multiple of 8 regions), one block scan per 4096 flags, emitted from registers
  for (int64_t i0 = lo; i0 < hi; i0 += (int64_t)kCompactThreads * 16) {
    const int64_t st = i0 + (int64_t)threadIdx.x * 16;
    uint32_t w[4] = {0u, 0u, 0u, 0u};
    if (st + 16 <= hi) {
      const uint2 a = *reinterpret_cast<const uint2*>(flags + st);
      const uint2 b = *reinterpret_cast<const uint2*>(flags + st + 8);
      w[0] = a.x; w[1] = a.y; w[2] = b.x; w[3] = b.y;
    } else {
      for (int k = 0; k < 16 && st + k < hi; ++k) w[k >> 2] |= (uint32_t)flags[st + k] << (8 * (k & 3));
    }
    const int c = __popc(w[0]) + __popc(w[1]) + __popc(w[2]) + __popc(w[3]);   // flags are 0/1 bytes
    int total;
    long long pos = base + block_exclusive_scan(c, warp_s, &total);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint32_t m = w[q];
      while (m) {  // set bytes in ascending order
        list[pos++] = rid_offset + st + q * 4 + ((__ffs(m) - 1) >> 3);
        m &= m - 1;
      }
    }
    base += total;
    __syncthreads();  // warp_s reuse
  }
}

static void scatter_grid(int64_t nblocks, int& grid, int& per_block) {
  grid = (int)(nblocks < 64 ? nblocks : 64);
  if (grid < 1) grid = 1;
  per_block = (int)((nblocks + grid - 1) / grid);
  grid = (int)((nblocks + per_block - 1) / per_block);
}

// ---------------------------------------------------------------------------
// Every tile of the EM x EN grid that a failed RM x RN region overlaps (a region may hold several tiles --
// 128x128 regions as two 128x64 slices -- or a tile several regions -- 32x32 regions in a 128x64 slice).
__global__ void tile_mark_kernel(const int64_t* __restrict__ list, const int64_t* __restrict__ d_n,
                                 int64_t rid_offset, int64_t Q, int64_t tiles_per_row, int RM, int RN, int EM, int EN,
                                 uint8_t* __restrict__ tile_flags) {
  const int64_t n = *d_n;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t rid = list[i] - rid_offset;
    const int64_t p = rid / Q, q = rid - p * Q;
    const int64_t r0 = p * RM / EM, r1 = (p * RM + RM - 1) / EM;
    const int64_t c0 = q * RN / EN, c1 = (q * RN + RN - 1) / EN;
    for (int64_t r = r0; r <= r1; ++r)
      for (int64_t c = c0; c <= c1; ++c) tile_flags[r * tiles_per_row + c] = 1;  // idempotent plain store
  }
}

// ---------------------------------------------------------------------------
// Recovery pairing (a10): the ascending failed list (128x128 regions or
// de-duplicated 128x128 tiles) is cut into tasks of one or two entries of the same
// 128-row band, so one CTA re-executes both with ONE A row panel staged for a
// 128x256 tcgen05 tile (B gathered from the two column panels): 6 MiB of operand
// reads per two regions instead of 8 MiB, and half the CTAs.  Inside each run of
// equal rows, entries at even offsets from the run start head a task; a head takes
// its successor when it lies in the same row.  Pairing is used only when there are
// more entries than SMs (otherwise one entry per CTA finishes sooner).
// tasks[t] = (list index << 1) | paired.  G = 4 (128x64 slices of 32x32 regions): up to
// min(4, max(2, ceil(n / #SM))) entries of one row per task, tasks[t] = (list index << 2) | (count - 1).  One CTA of 1024 threads, chunked scans.
constexpr int kPairThreads = 1024;

__device__ __forceinline__ int64_t block_scan_max_i64(int64_t v, int64_t* s_warp, int64_t* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int64_t y = __shfl_up_sync(0xFFFFFFFFu, v, o);
    if (lane >= o) v = v > y ? v : y;
  }
  if (lane == 31) s_warp[wid] = v;
  __syncthreads();
  if (wid == 0) {
    int64_t x = s_warp[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t y = __shfl_up_sync(0xFFFFFFFFu, x, o);
      if (lane >= o) x = x > y ? x : y;
    }
    s_warp[lane] = x;
  }
  __syncthreads();
  if (wid > 0) {
    const int64_t y = s_warp[wid - 1];
    v = v > y ? v : y;
  }
  *total = s_warp[31];
  __syncthreads();
  return v;
}

__device__ __forceinline__ int block_scan_excl_sum(int v, int* s_warp, int* total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xFFFFFFFFu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    int t = s_warp[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xFFFFFFFFu, t, o);
      if (lane >= o) t += y;
    }
    s_warp[lane] = t;
  }
  __syncthreads();
  const int r = (wid > 0 ? s_warp[wid - 1] : 0) + x - v;
  *total = s_warp[31];
  __syncthreads();
  return r;
}

constexpr int kPairPer = 4;  // entries per thread per block pass (4096 per pass: fewer block scans)

__global__ void __launch_bounds__(kPairThreads) pair_tasks_kernel(const int64_t* __restrict__ list,
                                                                  const int64_t* __restrict__ d_n, int64_t off,
                                                                  int64_t div, int64_t min_pair, int G, int grid,
                                                                  int lpt, int64_t* __restrict__ d_rec,
                                                                  int64_t rec_num, int64_t rec_den,
                                                                  int32_t* __restrict__ tasks_tmp,
                                                                  int32_t* __restrict__ tasks,
                                                                  int64_t* __restrict__ d_ntasks) {
  __shared__ int64_t s_max[32];
  __shared__ int s_sum[32];
  __shared__ int64_t s_incl[kPairThreads];
  // the re-execution grid that follows may start its prologue now (it waits for this grid to finish)
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int64_t n = *d_n;
  if (d_rec && threadIdx.x == 0) *d_rec = n * rec_num / rec_den;  // regions the re-execution will rewrite
  const bool pairing = n > min_pair;
  const int sh = G == 4 ? 2 : 1;
  // slice grouping (G = 4): as many entries per task as it takes to fill the SMs once, 2..4
  // (300 failed slices on 148 SMs: tasks of 3 -> one wave of N = 192, not 75 tasks of N = 256)
  if (G == 4 && pairing) {
    const int64_t need = (n + min_pair - 1) / min_pair;
    G = need < 2 ? 2 : (need > 4 ? 4 : (int)need);
  }
  int64_t carry_ls = -1;  // index of the last run start seen so far
  int64_t carry_t = 0;    // tasks emitted so far
  for (int64_t base = 0; base < n; base += (int64_t)kPairThreads * kPairPer) {
    const int64_t i0 = base + (int64_t)threadIdx.x * kPairPer;
    int64_t rows[kPairPer];
    bool rh[kPairPer];
    int64_t prev = (i0 > 0 && i0 - 1 < n) ? (list[i0 - 1] - off) / div : -2;
    int64_t lmax = -1;  // last run start among this thread's entries
#pragma unroll
    for (int j = 0; j < kPairPer; ++j) {
      const int64_t i = i0 + j;
      rows[j] = i < n ? (list[i] - off) / div : -1;
      rh[j] = i < n && rows[j] != prev;
      if (rh[j]) lmax = i;
      prev = rows[j];
    }
    int64_t blk_max;
    s_incl[threadIdx.x] = block_scan_max_i64(lmax, s_max, &blk_max);
    __syncthreads();
    int64_t ls = threadIdx.x ? s_incl[threadIdx.x - 1] : -1;  // last run start before this thread's entries
    ls = ls > carry_ls ? ls : carry_ls;
    int32_t w[kPairPer];
    int nh = 0;
#pragma unroll
    for (int j = 0; j < kPairPer; ++j) {
      const int64_t i = i0 + j;
      if (rh[j]) ls = i;
      if (i < n && (!pairing || ((i - ls) % G) == 0)) {
        int cnt = 1;  // entries of this task: the head and its successors in the same row, at most G
        if (pairing)
          for (int k = 1; k < G && i + k < n && (list[i + k] - off) / div == rows[j]; ++k) ++cnt;
        w[nh++] = (int32_t)((i << sh) | (cnt - 1));
      }
    }
    int tot;
    const int idx = block_scan_excl_sum(nh, s_sum, &tot);
    for (int k = 0; k < nh; ++k) tasks_tmp[carry_t + idx + k] = w[k];
    carry_t += tot;
    carry_ls = blk_max > carry_ls ? blk_max : carry_ls;
  }
  // Static LPT-like schedule for the persistent re-execution grid (CTA c runs positions c, c + grid, ...):
  // tasks sorted by entry count, largest first (stable), dealt round by round; the LAST round goes
  // forward (it may be partial and must land on CTAs 0..L-1) and the rounds alternate direction
  // backwards from it, so a CTA that got a small task in one round gets a large one in the next.
  const int64_t T = carry_t;
  const int mask = (1 << sh) - 1;
  __shared__ int s_cls[5], s_off[5];
  if (threadIdx.x < 5) s_cls[threadIdx.x] = 0;
  __syncthreads();
  for (int64_t i = threadIdx.x; i < T; i += kPairThreads) atomicAdd(&s_cls[(tasks_tmp[i] & mask) + 1], 1);
  __syncthreads();
  if (threadIdx.x == 0) {  // start of each size class in the sorted order (larger classes first)
    int acc = 0;
    for (int c = 4; c >= 1; --c) {
      s_off[c] = acc;
      acc += s_cls[c];
    }
  }
  __syncthreads();
  const int64_t nr = (T + grid - 1) / grid;
  for (int64_t base = 0; base < T; base += kPairThreads) {
    const int64_t i = base + threadIdx.x;
    const int32_t w = i < T ? tasks_tmp[i] : 0;
    const int c = i < T ? (w & mask) + 1 : 0;
    // stable rank inside the size class (one ballot-based block scan over the 4 class flags at once:
    // each class's count fits 10 bits of a packed 64-bit word)
    const unsigned long long f = c ? (1ull << (16 * (c - 1))) : 0ull;
    unsigned long long x = f;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(0xFFFFFFFFu, x, o);
      if (lane >= o) x += y;
    }
    __shared__ unsigned long long s_w[32];
    if (lane == 31) s_w[wid] = x;
    __syncthreads();
    if (wid == 0) {
      unsigned long long t = s_w[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(0xFFFFFFFFu, t, o);
        if (lane >= o) t += y;
      }
      s_w[lane] = t;
    }
    __syncthreads();
    const unsigned long long excl = (wid ? s_w[wid - 1] : 0ull) + x - f;
    const unsigned long long tot = s_w[31];
    if (i < T) {
      const int rank = (int)((excl >> (16 * (c - 1))) & 0xFFFFull);
      const int64_t srt = s_off[c] + rank;  // position in the sorted order
      const int64_t r = srt / grid, k = srt - r * grid;
      const int64_t cta = ((nr - 1 - r) & 1) ? (grid - 1 - k) : k;
      tasks[lpt ? r * grid + cta : i] = w;
    }
    __syncthreads();
    if (threadIdx.x < 4) s_off[threadIdx.x + 1] += (int)((tot >> (16 * threadIdx.x)) & 0xFFFFull);
    __syncthreads();
  }
  if (threadIdx.x == 0) *d_ntasks = T;
}

__global__ void hash_header_kernel(uint32_t* ck, uint32_t cap, uint32_t seed, uint32_t max_evict) {
  HashHeader* h = reinterpret_cast<HashHeader*>(ck);
  h->cap = cap;
  h->seed = seed;
  h->lock = 0;
  h->error = 0;
  h->collisions = 0ull;
  h->stash_n = 0;
  h->rehashes = 0;
  h->max_evict = max_evict;
}

// Cuckoo rehash (L270: "When a cycle is detected, the cuckoo hash table performs hash
// tables rehashing"; Reading R24).  Runs after every protected / recovery run of a cuckoo
// store and returns at once while the stash is empty.  Otherwise, per attempt: a new seed
// (new H1, H2); the stash is copied to shared memory and emptied; every thread walks a
// strided share of T1/T2 and takes out (one 128-bit exchange) each entry that is not at
// its slot under the new seed, re-placing it with the ordinary eviction walk; then the old
// stash entries are placed.  Walks place entries only at their new-seed slots, so after
// the pass every entry sits at H1'/H2' -- or, if a walk hit the bound, in the stash again,
// and the next attempt tries another seed.  Rehash walks use the default bound and do not
// count as insertion collisions (Table II counts inserts).
constexpr int kRehashAttempts = 16;
__global__ void __launch_bounds__(1024) cuckoo_rehash_kernel(uint32_t* ck) {
  HashHeader* hdr = reinterpret_cast<HashHeader*>(ck);
  __shared__ uint4 s_stash[kCuckooStash];
  __shared__ uint32_t s_n, s_seed, s_more;
  __shared__ unsigned long long s_coll;
  // loop control is decided by thread 0 (an atomic read of the stash count at gpu scope) and shared, so every
  // thread takes the same number of attempts (a per-thread read could see a stale value and split the CTA
  // across the __syncthreads below)
  if (threadIdx.x == 0) s_more = atomicAdd(&hdr->stash_n, 0u);
  __syncthreads();
  if (s_more == 0) return;
  uint4* tab = reinterpret_cast<uint4*>(ck + sizeof(HashHeader) / 4);
  const uint32_t cap = hdr->cap;
  if (threadIdx.x == 0) s_coll = hdr->collisions;
  for (int attempt = 0; attempt < kRehashAttempts; ++attempt) {
    __syncthreads();
    if (threadIdx.x == 0) {
      const uint32_t n = hdr->stash_n;
      s_n = n < (uint32_t)kCuckooStash ? n : (uint32_t)kCuckooStash;
      s_seed = hash_fmix32(hdr->seed + 0x9E3779B9u, 0x5BD1E995u + (uint32_t)attempt);
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < s_n; i += blockDim.x) s_stash[i] = tab[2ull * cap + i];
    __syncthreads();
    if (threadIdx.x == 0) {
      hdr->seed = s_seed;
      hdr->stash_n = 0;
      hdr->rehashes += 1;
      __threadfence();
    }
    __syncthreads();
    const uint32_t seed = s_seed;
    const uint4 empty = make_uint4(kEmptyKey, kEmptyKey, kEmptyKey, kEmptyKey);
    for (uint64_t s = threadIdx.x; s < 2ull * cap; s += blockDim.x) {
      const int t = s < cap ? 0 : 1;
      const uint32_t i = (uint32_t)(s - (uint64_t)t * cap);
      const uint32_t key = *reinterpret_cast<volatile uint32_t*>(tab + s);
      if (key == kEmptyKey || cuckoo_h(t, key, seed, cap) == i) continue;
      const uint4 e = atom_exch_128(tab + s, empty);
      if (e.x != kEmptyKey) cuckoo_place(hdr, tab, cap, seed, e, kCuckooMaxEvict, false);
    }
    for (uint32_t i = threadIdx.x; i < s_n; i += blockDim.x) cuckoo_place(hdr, tab, cap, seed, s_stash[i], kCuckooMaxEvict, false);
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_more = atomicAdd(&hdr->stash_n, 0u);
    __syncthreads();
    if (s_more == 0) break;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    hdr->collisions = s_coll;
    if (hdr->stash_n) hdr->error = 1u;   // no seed found: the stash still holds entries (LP_ERR_CAPACITY)
  }
}

__global__ void stats_kernel(const uint32_t* ck, int has_hash, int64_t* d_stats) {
  if (has_hash) {
    const HashHeader* h = reinterpret_cast<const HashHeader*>(ck);
    d_stats[0] = (int64_t)h->collisions;
    d_stats[1] = (int64_t)h->error;
  } else {
    d_stats[0] = 0;
    d_stats[1] = 0;
  }
}

// Crash injection (harness; Reading R11).  One block per injected region.
template <int S>
__global__ void inject_kernel(uint8_t* out, int64_t ldc_bytes, int64_t Q, int RM, int row_bytes,
                              const uint8_t* stale, uint32_t* ck, int store, const int64_t* rids, int64_t rid_offset,
                              int64_t R, uint32_t mode, uint64_t seed) {
  const int64_t grid = rids[blockIdx.x];
  const int64_t r = grid - rid_offset;
  if (r < 0 || r >= R) return;  // not a region of this shard (rids are global): nothing to corrupt
  const int64_t p = r / Q, q = r - p * Q;
  const int64_t base = p * (int64_t)RM * ldc_bytes + q * (int64_t)row_bytes;
  const int wpr = row_bytes / 4;
  const int words = RM * wpr;
  const uint64_t h = mix64(seed ^ (0xD1B54A32D192ED03ull * (uint64_t)(grid + 1)));
  if (mode == 0 || mode == 1) {  // stale words / stale region
    const int m = mode == 1 ? words : 1 + (int)(h % (uint64_t)words);
    const int start = mode == 1 ? 0 : (int)((h >> 32) % (uint64_t)words);
    for (int i = threadIdx.x; i < m; i += blockDim.x) {
      const int wi = (start + i) % words;
      const int64_t off = base + (int64_t)(wi / wpr) * ldc_bytes + (wi % wpr) * 4;
      *reinterpret_cast<uint32_t*>(out + off) = *reinterpret_cast<const uint32_t*>(stale + off);
    }
  } else if (mode == 2) {  // bit flip
    if (threadIdx.x == 0) {
      const int wi = (int)(h % (uint64_t)words);
      const int bit = (int)((h >> 40) & 31u);
      const int64_t off = base + (int64_t)(wi / wpr) * ldc_bytes + (wi % wpr) * 4;
      *reinterpret_cast<uint32_t*>(out + off) ^= (1u << bit);
    }
  } else {  // stale record
    if (threadIdx.x == 0) {
      if (store == 0) {
        for (int s = 0; s < S; ++s) ck[r * S + s] = kSentinel;
      } else if (store >= 3) {
        const HashHeader* hdr = reinterpret_cast<const HashHeader*>(ck);
        uint4* tab = reinterpret_cast<uint4*>(ck + sizeof(HashHeader) / 4);
        for (int t = 0; t < 2; ++t) {
          uint4* e = tab + (uint64_t)t * hdr->cap + cuckoo_h(t, (uint32_t)grid, hdr->seed, hdr->cap);
          if (e->x == (uint32_t)grid) {
            e->y = kSentinel;
            e->z = kSentinel;
            e->w = kSentinel;
            break;
          }
        }
      } else {
        const HashHeader* hdr = reinterpret_cast<const HashHeader*>(ck);
        uint32_t* ent = ck + sizeof(HashHeader) / 4;
        const uint32_t cap = hdr->cap;
        const uint32_t home = hash_fmix32((uint32_t)grid, hdr->seed) % cap;
        for (uint32_t i = 0; i < cap; ++i) {
          const uint32_t slot = (uint32_t)(((uint64_t)home + (uint64_t)i * i) % cap);
          uint32_t* e = ent + (uint64_t)slot * (1 + S);
          if (e[0] == (uint32_t)grid) {
            for (int s = 0; s < S; ++s) e[1 + s] = kSentinel;
            break;
          }
          if (e[0] == kEmptyKey) break;
        }
      }
    }
  }
}

}  // namespace

// ===========================================================================
cudaError_t launch_cksum_init(void* ck, size_t bytes, const HashInfo& hi, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(ck, 0xFF, bytes, st);
  if (e != cudaSuccess) return e;
  if (hi.store != 0) {
    hash_header_kernel<<<1, 1, 0, st>>>((uint32_t*)ck, hi.cap, hi.seed, hi.max_evict);
    e = cudaGetLastError();
  }
  return e;
}

// Strip width: G regions per warp.  G = 32 / cpr makes one warp load instruction
// cover one row of the whole strip (512 B contiguous); it is halved while that
// would leave fewer than kValMinWarps warp tasks (too few bytes in flight: 128x128
// bf16 regions at G = 2 leave 2048 warps / 8 MiB in flight and measure 28.7 us
// for 128 MiB vs 22.5 us at G = 1).  LP_VALIDATE_G=<log2> overrides (A/B runs).
constexpr int64_t kValMinWarps = 4096;

// output size from which Adler validation uses the 3-CTA/SM build (LP_VAL_ADLER_BIG=<MiB> for A/B runs)
static uint64_t val_adler_big_bytes() {
  static const uint64_t v = [] {
    const char* e = getenv("LP_VAL_ADLER_BIG");
    return (uint64_t)(e ? atoll(e) : 512) << 20;
  }();
  return v;
}

static ValLaunch plan_validate(const RegionGeom& g, int sm_count) {
  ValLaunch L;
  const int cpr = (g.RN * g.es) / 16;
  int gl = 0;
  while ((2 << gl) * cpr <= 32) ++gl;                  // G * cpr <= 32
  while (gl > 0 && (g.R >> gl) < kValMinWarps) --gl;
  static const int g_override = [] {  // LP_VALIDATE_G=<log2>: A/B override, read once per process
    const char* e = getenv("LP_VALIDATE_G");
    const int v = e ? atoi(e) : -1;
    return (v >= 0 && v <= 5) ? v : -1;
  }();
  if (g_override >= 0) gl = g_override;
  L.g_log2 = gl;
  const int64_t unit = (int64_t)kValWarps << gl;
  int64_t max_ctas = (int64_t)sm_count * 16;
  if (max_ctas > kMaxValCtas) max_ctas = kMaxValCtas;  // per-CTA counts live in the caller's workspace
  int64_t ctas = (g.R + unit - 1) / unit;
  if (ctas > max_ctas) ctas = max_ctas;
  if (ctas < 1) ctas = 1;
  int64_t rpc = (g.R + ctas - 1) / ctas;
  rpc = (rpc + unit - 1) / unit * unit;
  ctas = (g.R + rpc - 1) / rpc;
  L.rpc = rpc;
  L.grid = dim3((unsigned)(ctas < 1 ? 1 : ctas));
  return L;
}

size_t validate_counts_bytes(const RegionGeom& g, int sm_count) {
  (void)g;
  return (size_t)sm_count * 16 * sizeof(uint32_t) + 256;
}

// Re-validation split around a recovery (lp_recover_revalidate; array table): the regions the previous validate
// did NOT flag are re-validated beside the recovery (MODE 4: flags = skip mask, mismatches counted), the flagged
// ones -- the failed list -- after it, one warp per region.  Together: every region of the final state checked.
cudaError_t launch_validate_skip_count(const RegionGeom& g, uint32_t mask, const void* out, const void* ck,
                                       const uint8_t* flags, unsigned long long* d_count, int sm_count,
                                       cudaStream_t st) {
  const int row_bytes = g.RN * g.es;
  const int cpr = row_bytes / 16;
  int cpr_log2 = 0;
  while ((1 << cpr_log2) < cpr) ++cpr_log2;
  const ValLaunch L = plan_validate(g, sm_count);
  const int mb = ((mask & kAdler) != 0 && (uint64_t)g.R * (uint64_t)g.RM * (uint64_t)row_bytes >= val_adler_big_bytes())
                     ? LP_VAL_ADLER_MINB : 4;
  const NvlsCount nv{nullptr, nullptr, 1};
  const uint8_t* o = (const uint8_t*)out;
  const int64_t ldcb = g.ldc * g.es;
  cudaError_t e;
  switch (mask) {
#define LP_VCASE(M)                                                                                          \
  case M:                                                                                                    \
    e = validate_dispatch_mode<M>(4, mb, L, st, o, ldcb, g.Q, g.R, g.RM, row_bytes, cpr_log2,                   \
                                  (const uint32_t*)ck, g.rid_offset, const_cast<uint8_t*>(flags), nullptr,      \
                                  nullptr, nullptr, nullptr, reinterpret_cast<int64_t*>(d_count), nv);          \
    break;
    LP_VCASE(1)
    LP_VCASE(2)
    LP_VCASE(3)
    LP_VCASE(4)
    LP_VCASE(5)
    LP_VCASE(6)
    LP_VCASE(7)
#undef LP_VCASE
    default:
      return cudaErrorInvalidValue;
  }
  return e;
}

namespace {
// One warp per listed region (global rid list[i]): record of the stored words vs the array table entry;
// mismatches added to *d_count.
template <uint32_t MASK>
__global__ void __launch_bounds__(256) validate_list_count_kernel(const uint8_t* __restrict__ out, int64_t ldc_bytes,
                                                                  int64_t Q, int RM, int row_bytes, int cpr_log2,
                                                                  const uint32_t* __restrict__ ck, int64_t rid_offset,
                                                                  const int64_t* __restrict__ list,
                                                                  const int64_t* __restrict__ d_n,
                                                                  unsigned long long* __restrict__ d_count) {
  constexpr int S = selem_of(MASK);
  const int lane = threadIdx.x & 31;
  const int64_t n = *d_n;
  const int chunks = RM << cpr_log2, cmask = (1 << cpr_log2) - 1;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += warps) {
    const int64_t r = list[i] - rid_offset, p = r / Q, q = r - p * Q;
    const uint8_t* base = out + p * (int64_t)RM * ldc_bytes + q * (int64_t)row_bytes;
    CkPartial<MASK> part;
    for (int c = lane; c < chunks; c += 32) {
      const uint4 v = ld_stream_u4(base + (int64_t)(c >> cpr_log2) * ldc_bytes + ((c & cmask) << 4));
      part.add4(v.x, v.y, v.z, v.w, (uint32_t)((c >> cpr_log2) * row_bytes + ((c & cmask) << 4) + 1));
    }
    const CkRecord rec = warp_reduce<MASK>(part);
    if (lane == 0) {
      uint32_t w[3];
      record_words<MASK>(rec, (uint64_t)RM * (uint64_t)row_bytes, w);
      bool bad = false;
#pragma unroll
      for (int s2 = 0; s2 < S; ++s2) bad |= (ck[r * S + s2] != w[s2]);
      if (bad) atomicAdd(d_count, 1ull);
    }
  }
}
}  // namespace

cudaError_t launch_validate_list_count(const RegionGeom& g, uint32_t mask, const void* out, const void* ck,
                                       const int64_t* list, const int64_t* d_n, unsigned long long* d_count,
                                       int sm_count, cudaStream_t st) {
  const int row_bytes = g.RN * g.es;
  const int cpr = row_bytes / 16;
  int cpr_log2 = 0;
  while ((1 << cpr_log2) < cpr) ++cpr_log2;
  const unsigned grid = (unsigned)(sm_count * 8);
  const uint8_t* o = (const uint8_t*)out;
  const int64_t ldcb = g.ldc * g.es;
  switch (mask) {
#define LP_LVCASE(M)                                                                                            \
  case M:                                                                                                       \
    validate_list_count_kernel<M><<<grid, 256, 0, st>>>(o, ldcb, g.Q, g.RM, row_bytes, cpr_log2,                 \
                                                        (const uint32_t*)ck, g.rid_offset, list, d_n, d_count); \
    break;
    LP_LVCASE(1)
    LP_LVCASE(2)
    LP_LVCASE(3)
    LP_LVCASE(4)
    LP_LVCASE(5)
    LP_LVCASE(6)
    LP_LVCASE(7)
#undef LP_LVCASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_validate(const RegionGeom& g, uint32_t mask, const HashInfo& hi, const void* out, const void* ck,
                            uint8_t* flags, uint32_t* records, int sm_count, cudaStream_t st, uint32_t* counts,
                            int64_t* list, int64_t* d_n, uint32_t* ticket, const NvlsCount* nvc) {
  const int row_bytes = g.RN * g.es;
  NvlsCount nv{nullptr, nullptr, 1};
  if (nvc && !records) nv = *nvc;
  const int cpr = row_bytes / 16;
  int cpr_log2 = 0;
  while ((1 << cpr_log2) < cpr) ++cpr_log2;
  const int mode = records ? 2 : (hi.store == 0 ? 0 : (hi.store <= 2 ? 1 : 3));
  const ValLaunch L = plan_validate(g, sm_count);
  // Adler records on large outputs: the 80-register build (3 CTAs/SM; the 64-register one spills ~100 B/thread)
  const int mb = ((mask & kAdler) != 0 && (uint64_t)g.R * (uint64_t)g.RM * (uint64_t)row_bytes >= val_adler_big_bytes())
                     ? LP_VAL_ADLER_MINB : 4;
  const bool fuse = !records && ticket && g.R <= kFusedCompactMaxR;
  uint32_t* tk = fuse ? ticket : nullptr;
  const uint8_t* o = (const uint8_t*)out;
  const int64_t ldcb = g.ldc * g.es;
  cudaError_t e;
  switch (mask) {
#define LP_VCASE(M)                                                                                          \
  case M:                                                                                                    \
    e = validate_dispatch_mode<M>(mode, mb, L, st, o, ldcb, g.Q, g.R, g.RM, row_bytes, cpr_log2,                \
                                  (const uint32_t*)ck, g.rid_offset, flags, records, counts, tk, list, d_n, nv);\
    break;
    LP_VCASE(1)
    LP_VCASE(2)
    LP_VCASE(3)
    LP_VCASE(4)
    LP_VCASE(5)
    LP_VCASE(6)
    LP_VCASE(7)
#undef LP_VCASE
    default:
      return cudaErrorInvalidValue;
  }
  if (e != cudaSuccess || records || fuse) return e;
  // ordered compaction: one pass, offsets from the validate kernel's per-CTA counts
  int sg, per;
  scatter_grid(L.grid.x, sg, per);
  // programmatic dependent launch: the scatter grid's launch overlaps the validate grid
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)sg);
  cfg.blockDim = dim3(kCompactThreads);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, compact_scatter_kernel, (const uint8_t*)flags, (int64_t)g.R,
                            (const uint32_t*)counts, (int)L.grid.x, (int64_t)L.rpc, per, (int64_t)g.rid_offset,
                            list, d_n, nv);
}

size_t compact_scratch_bytes(int64_t R) {
  const int64_t nb = (R + kCompactChunk - 1) / kCompactChunk;
  return (size_t)(nb > 0 ? nb : 1) * sizeof(uint32_t);
}

cudaError_t launch_compact(const RegionGeom& g, const uint8_t* flags, uint32_t* block_counts, int64_t* list,
                           int64_t* d_n, cudaStream_t st) {
  int64_t nb = (g.R + kCompactChunk - 1) / kCompactChunk;
  if (nb < 1) nb = 1;
  compact_count_kernel<<<(unsigned)nb, kCompactThreads, 0, st>>>(flags, g.R, block_counts);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  int sg, per;
  scatter_grid(nb, sg, per);
  compact_scatter_kernel<<<sg, kCompactThreads, 0, st>>>(flags, g.R, block_counts, (int)nb, kCompactChunk, per,
                                                         g.rid_offset, list, d_n, NvlsCount{nullptr, nullptr, 1});
  return cudaGetLastError();
}

cudaError_t launch_inject(const RegionGeom& g, uint32_t mask, const HashInfo& hi, void* out, void* ck,
                          const void* stale, const int64_t* rids, int64_t n, uint32_t mode, uint64_t seed,
                          cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  const int S = selem_of(mask);
  const int row_bytes = g.RN * g.es;
#define LP_ICASE(SV)                                                                                           \
  inject_kernel<SV><<<(unsigned)n, 256, 0, st>>>((uint8_t*)out, g.ldc * g.es, g.Q, g.RM, row_bytes,           \
                                                 (const uint8_t*)stale, (uint32_t*)ck, hi.store, rids,        \
                                                 g.rid_offset, g.R, mode, seed)
  if (S == 1) LP_ICASE(1);
  else if (S == 2) LP_ICASE(2);
  else LP_ICASE(3);
#undef LP_ICASE
  return cudaGetLastError();
}

cudaError_t launch_tiles_of_failed(const RegionGeom& g, int EM, int EN, const int64_t* list, const int64_t* d_n,
                                   uint8_t* tile_flags, int64_t T, uint32_t* block_counts, int64_t* tile_list,
                                   int64_t* d_ntiles, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(tile_flags, 0, (size_t)T, st);
  if (e != cudaSuccess) return e;
  tile_mark_kernel<<<(unsigned)(g.R < 148 * 4 * 256 ? (g.R + 255) / 256 : 148 * 4), 256, 0, st>>>(
      list, d_n, g.rid_offset, g.Q, g.N / EN, g.RM, g.RN, EM, EN, tile_flags);
  e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  RegionGeom tg = g;
  tg.R = T;
  tg.rid_offset = 0;
  return launch_compact(tg, tile_flags, block_counts, tile_list, d_ntiles, st);
}

__global__ void scale_count_kernel(const int64_t* __restrict__ src, int64_t num, int64_t den,
                                   int64_t* __restrict__ dst) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  *dst = *src * num / den;
}

cudaError_t launch_scale_count(const int64_t* src, int64_t num, int64_t den, int64_t* dst, cudaStream_t st) {
  scale_count_kernel<<<1, 1, 0, st>>>(src, num, den, dst);
  return cudaGetLastError();
}

cudaError_t launch_pair_tasks(const int64_t* list, const int64_t* d_n, int64_t off, int64_t div, int64_t min_pair,
                              int G, int grid, int32_t* tasks_tmp, int32_t* tasks, int64_t* d_ntasks,
                              int64_t* d_rec, int64_t rec_num, int64_t rec_den, cudaStream_t st) {
  static const int lpt = [] {  // LP_TASK_ORDER=row keeps the grouping's row order (A/B runs)
    const char* e = getenv("LP_TASK_ORDER");
    return (e && e[0] == 'r') ? 0 : 1;
  }();
  pair_tasks_kernel<<<1, kPairThreads, 0, st>>>(list, d_n, off, div, min_pair, G, grid < 1 ? 1 : grid, lpt, d_rec,
                                                rec_num, rec_den < 1 ? 1 : rec_den, tasks_tmp, tasks, d_ntasks);
  return cudaGetLastError();
}

cudaError_t launch_cuckoo_rehash(void* ck, cudaStream_t st) {
  cuckoo_rehash_kernel<<<1, 1024, 0, st>>>((uint32_t*)ck);
  return cudaGetLastError();
}

cudaError_t launch_stats(const HashInfo& hi, const void* ck, int64_t* d_stats, cudaStream_t st) {
  stats_kernel<<<1, 1, 0, st>>>((const uint32_t*)ck, hi.store != 0 ? 1 : 0, d_stats);
  return cudaGetLastError();
}

}  // namespace lp
