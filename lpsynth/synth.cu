// lpsynth/synth.cu -- device twin of lpsynth/gen.py (seeded counter-based inputs).
//
// Holds none of the Lazy-Persistency arithmetic; it only materialises workload
// inputs in HBM so that 8 GiB operands never cross
// PCIe. Bit-exact agreement with gen.py is a -m gpu test.
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
  z += kGolden;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__device__ __forceinline__ float value_of(uint64_t x, int kind) {
  switch (kind) {
    case 0: return (float)((double)(x >> 40) * (1.0 / 8388608.0) - 1.0);
    case 1: return (float)((int)(x % 5ull) - 2);
    default: return (float)((int)(x % 17ull) - 8);
  }
}

__global__ void synth_fill_kernel(void* dst, int64_t rows, int64_t cols, int64_t ld, int64_t row0,
                                  int64_t ncols_global, uint64_t seed, int kind, int dtype) {
  const int64_t total = rows * cols;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = e / cols, c = e - r * cols;
    const uint64_t x = splitmix64(seed * kGolden + (uint64_t)(row0 + r) * (uint64_t)ncols_global + (uint64_t)c);
    const int64_t off = r * ld + c;
    if (kind == 3) {  // bits
      if (dtype == 1) ((uint16_t*)dst)[off] = (uint16_t)(x & 0xFFFFu);
      else ((uint32_t*)dst)[off] = (uint32_t)(x & 0xFFFFFFFFu);
      continue;
    }
    const float v = value_of(x, kind);
    if (dtype == 1) ((__nv_bfloat16*)dst)[off] = __float2bfloat16_rn(v);
    else if (dtype == 3) ((int32_t*)dst)[off] = (int32_t)v;
    else ((float*)dst)[off] = v;
  }
}

}  // namespace

extern "C" int synth_fill(void* dst, int64_t rows, int64_t cols, int64_t ld, int64_t row0,
                          int64_t ncols_global, uint64_t seed, int kind, int dtype, void* stream) {
  if (!dst || rows < 0 || cols < 0 || ld < cols || kind < 0 || kind > 3 || dtype < 0 || dtype > 3) return 1;
  if (dtype == 3 && kind == 0) return 1;  // int32 inputs are integer-valued kinds
  if (rows == 0 || cols == 0) return 0;
  const int64_t total = rows * cols;
  int64_t blocks = (total + 255) / 256;
  if (blocks > 148 * 64) blocks = 148 * 64;
  synth_fill_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(dst, rows, cols, ld, row0, ncols_global,
                                                                         seed, kind, dtype);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

// ---- SpMV structure (twin of lpsynth/csr.py columns()): one warp per row.
namespace {
constexpr int64_t kBandStride = 8;

__global__ void synth_csr_cols_kernel(const int64_t* __restrict__ rp, int64_t rows, int64_t row0, int64_t ncols,
                                      uint64_t seed, int32_t* __restrict__ cols) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < rows; i += warps) {
    const int64_t b = rp[i], e = rp[i + 1], len = e - b, r = row0 + i;
    const int64_t base = r - (len * kBandStride) / 2;
    for (int64_t k = lane; k < len; k += 32) {
      const uint64_t h = splitmix64(seed * kGolden + (uint64_t)(b + k));
      int64_t c = (base + k * kBandStride + (int64_t)(h % (uint64_t)kBandStride)) % ncols;
      if (c < 0) c += ncols;
      cols[b - rp[0] + k] = (int32_t)c;
    }
  }
}
}  // namespace

// cols[0 .. rp[rows]-rp[0]) for rows [row0, row0+rows) given their device row_ptr slice rp[0..rows].
extern "C" int synth_csr_cols(const int64_t* rp, int64_t rows, int64_t row0, int64_t ncols, uint64_t seed,
                              int32_t* cols, void* stream) {
  if (!rp || !cols || rows < 0 || ncols <= 0) return 1;
  if (rows == 0) return 0;
  int64_t blocks = (rows + 7) / 8;
  if (blocks > 148 * 32) blocks = 148 * 32;
  synth_csr_cols_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(rp, rows, row0, ncols, seed, cols);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
