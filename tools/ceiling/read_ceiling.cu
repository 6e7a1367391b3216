// read_ceiling.cu -- measurement tooling (not part of liblp): the plain streaming read-reduce
// ceiling the validate kernel is compared against.  Every CTA of a
// grid-stride loop reads 16-B non-allocating vectors, 8 in flight per thread, XOR-folds them
// and writes one word per CTA (so the loads cannot be elided).
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -shared -Xcompiler -fPIC -o libreadceil.so read_ceiling.cu
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ uint4 ld_nc(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__global__ void __launch_bounds__(256) read_xor_kernel(const uint4* __restrict__ p, int64_t n16, uint32_t* out) {
  uint32_t acc = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 7 * stride < n16; i += 8 * stride) {
    uint4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = ld_nc(p + i + u * stride);
#pragma unroll
    for (int u = 0; u < 8; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  for (; i < n16; i += stride) {
    const uint4 v = ld_nc(p + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  acc = __reduce_xor_sync(0xFFFFFFFFu, acc);
  if ((threadIdx.x & 31) == 0) atomicXor(out + blockIdx.x, acc);
}

extern "C" int read_ceiling(const void* buf, int64_t bytes, uint32_t* out, int ctas_per_sm, void* stream) {
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  read_xor_kernel<<<sms * ctas_per_sm, 256, 0, (cudaStream_t)stream>>>((const uint4*)buf, bytes / 16, out);
  return (int)cudaGetLastError();
}
