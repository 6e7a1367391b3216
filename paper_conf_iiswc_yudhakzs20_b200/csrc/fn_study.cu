// fn_study.cu -- false-negative rate of the LP checksums under random error injection
// (NEXT row N3; L53 "there is a small probability of false positive, i.e. the checksum
// indicates no persistency failure when in fact there is a failure"; L192 "through
// random error injection, modular and Adler-32 checksums both provide false negative
// rates of less than one in two billion ... [both] less than one in a trillion").
//
// A trial corrupts a region of `nwords` 32-bit words and asks whether each checksum
// set still matches.  The checksums are linear in the stored data, so only the changed
// words matter:
//   MOD   unchanged  <=>  sum (new_i - old_i) == 0            (mod 2^32)
//   XOR   unchanged  <=>  xor (new_i ^ old_i) == 0
//   ADLER unchanged  <=>  sum d_b == 0 and sum pos_b * d_b == 0  (mod 65521)
// with d_b the byte differences at 1-based byte positions pos_b (closed form of
// lp_device.cuh).  Region content, positions and new values come from a counter-based
// generator keyed by (seed, trial), so trials are reproducible; the first `dump`
// trials are written out for the CPU oracle to re-check from fully materialised regions.
//
// Corruption models (the paper does not define its injection; Reading R23):
//   0 RANDOM_WORDS  k in [1, kmax] words take fresh random values (stale data)
//   1 BITFLIPS      k in [1, kmax] single-bit flips
//   2 ADVERSARIAL   one bit b set in word i and cleared in word j (MOD and XOR blind)
//   3 ZEROED        k in [1, kmax] words revert to zero (never-written memory)
#include <cuda_runtime.h>
#include <stdint.h>

#include "lp_device.cuh"
#include "lp_internal.h"

namespace lp {
namespace {

constexpr int kMaxK = 8;

struct Rng {
  uint64_t s;
  __device__ __forceinline__ uint64_t next() {
    s += 0x9E3779B97F4A7C15ull;
    uint64_t z = s;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
  }
};

__device__ __forceinline__ int64_t mod_p(int64_t x) {
  int64_t r = x % 65521;
  return r < 0 ? r + 65521 : r;
}

// counts: [0] effective trials (region changed), [1] undetected MOD, [2] XOR,
// [3] MOD|XOR, [4] ADLER, [5] MOD|XOR|ADLER, [6] no-op trials
__global__ void fn_study_kernel(uint64_t seed, int64_t trials, int64_t nwords, int mode, int kmax,
                                unsigned long long* __restrict__ counts, uint32_t* __restrict__ dump,
                                int64_t dump_trials) {
  unsigned long long c[7] = {0, 0, 0, 0, 0, 0, 0};
  const uint64_t nbytes = (uint64_t)nwords * 4u;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < trials;
       t += (int64_t)gridDim.x * blockDim.x) {
    Rng rng{seed * 0xD1B54A32D192ED03ull + (uint64_t)t * 0x9E3779B97F4A7C15ull};
    int64_t pos[kMaxK];
    uint32_t oldw[kMaxK], neww[kMaxK];
    int k;
    if (mode == 2) {
      k = 2;
      const uint32_t bit = 1u << (rng.next() & 31u);
      pos[0] = (int64_t)(rng.next() % (uint64_t)nwords);
      do {
        pos[1] = (int64_t)(rng.next() % (uint64_t)nwords);
      } while (pos[1] == pos[0]);
      oldw[0] = (uint32_t)rng.next() & ~bit;  // bit clear, gets set
      oldw[1] = (uint32_t)rng.next() | bit;   // bit set, gets cleared
      neww[0] = oldw[0] | bit;
      neww[1] = oldw[1] & ~bit;
    } else {
      k = 1 + (int)(rng.next() % (uint64_t)kmax);
      int n = 0;
      for (int j = 0; j < k; ++j) {
        const int64_t p = (int64_t)(rng.next() % (uint64_t)nwords);
        int slot = -1;
        for (int i = 0; i < n; ++i)
          if (pos[i] == p) slot = i;
        if (slot < 0) {  // first touch of this word: draw its original content
          slot = n++;
          pos[slot] = p;
          oldw[slot] = (uint32_t)rng.next();
          neww[slot] = oldw[slot];
        }
        if (mode == 0)
          neww[slot] = (uint32_t)rng.next();
        else if (mode == 1)
          neww[slot] ^= 1u << (rng.next() & 31u);
        else
          neww[slot] = 0u;
      }
      k = n;
    }
    uint32_t dmod = 0, dxor = 0;
    int64_t ds = 0, dw = 0;
    bool changed = false;
    for (int i = 0; i < k; ++i) {
      changed |= (oldw[i] != neww[i]);
      dmod += neww[i] - oldw[i];
      dxor ^= neww[i] ^ oldw[i];
      for (int b = 0; b < 4; ++b) {
        const int64_t d = (int64_t)((neww[i] >> (8 * b)) & 0xFFu) - (int64_t)((oldw[i] >> (8 * b)) & 0xFFu);
        ds += d;
        dw = mod_p(dw + mod_p((int64_t)(((uint64_t)pos[i] * 4u + (uint64_t)b + 1u) % 65521u) * d));
      }
    }
    const bool um = changed && dmod == 0, ux = changed && dxor == 0;
    const bool ua = changed && mod_p(ds) == 0 && dw == 0;
    (void)nbytes;
    if (!changed) {
      c[6]++;
    } else {
      c[0]++;
      c[1] += um;
      c[2] += ux;
      c[3] += (um && ux);
      c[4] += ua;
      c[5] += (um && ux && ua);
    }
    if (t < dump_trials) {
      // [k, pos lo32 x8, old x8, new x8, detect bits (MOD, XOR, ADLER detected)]
      uint32_t* d = dump + t * 26;
      d[0] = (uint32_t)k;
      for (int i = 0; i < kMaxK; ++i) {
        d[1 + i] = i < k ? (uint32_t)pos[i] : 0u;
        d[9 + i] = i < k ? oldw[i] : 0u;
        d[17 + i] = i < k ? neww[i] : 0u;
      }
      d[25] = (changed ? 8u : 0u) | (um ? 0u : 1u) | (ux ? 0u : 2u) | (ua ? 0u : 4u);
    }
  }
  // warp-aggregate then one atomic per warp per counter
  for (int i = 0; i < 7; ++i) {
    unsigned long long v = c[i];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(&counts[i], v);
  }
}

}  // namespace

cudaError_t launch_fn_study(uint64_t seed, int64_t trials, int64_t nwords, int mode, int kmax,
                            unsigned long long* counts, uint32_t* dump, int64_t dump_trials, int sm_count,
                            cudaStream_t st) {
  if (kmax < 1 || kmax > kMaxK || nwords < 2 || mode < 0 || mode > 3) return cudaErrorInvalidValue;
  cudaError_t e = cudaMemsetAsync(counts, 0, 7 * sizeof(unsigned long long), st);
  if (e != cudaSuccess) return e;
  int64_t blocks = (trials + 255) / 256;
  if (blocks > (int64_t)sm_count * 16) blocks = (int64_t)sm_count * 16;
  if (blocks < 1) blocks = 1;
  fn_study_kernel<<<(unsigned)blocks, 256, 0, st>>>(seed, trials, nwords, mode, kmax, counts, dump, dump_trials);
  return cudaGetLastError();
}

}  // namespace lp
