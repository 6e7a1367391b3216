// Standalone check of the cluster-launch-control work loop used by tmm_tc4_kernel<..., CLC = true>:
// clusters of 2 CTAs, grid = 2 * T, a "producer" thread per CTA + 4 "epilogue" warps per CTA consume every
// response; the leader issues the next try_cancel.  count[t] must be 1 for every tile.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c) : "memory"); }
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void mbar_arrive(uint64_t* b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory"); }
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t par) {
  uint32_t done;
  do {
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(done) : "r"(smem_u32(b)), "r"(par) : "memory");
  } while (!done);
}
__device__ __forceinline__ uint32_t mapa0(const void* p) { uint32_t r; asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(smem_u32(p))); return r; }
__device__ __forceinline__ void arrive_remote(uint32_t a) { asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(a) : "memory"); }
__device__ __forceinline__ uint32_t ctarank() { uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r; }
__device__ __forceinline__ void cluster_sync() { asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory"); }
__device__ __forceinline__ void try_cancel(uint4* resp, uint64_t* bar) {
  asm volatile("clusterlaunchcontrol.try_cancel.async.shared::cta.mbarrier::complete_tx::bytes.multicast::cluster::all.b128 [%0], [%1];" ::"r"(smem_u32(resp)), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ long long decode(const uint4* resp) {
  uint32_t x, valid;
  asm volatile("{\n\t.reg .pred p;\n\t.reg .b128 r;\n\tld.shared.b128 r, [%2];\n\t"
               "clusterlaunchcontrol.query_cancel.is_canceled.pred.b128 p, r;\n\tselp.u32 %1, 1, 0, p;\n\tmov.u32 %0, 0;\n\t"
               "@p clusterlaunchcontrol.query_cancel.get_first_ctaid.v4.b32.b128 {%0, _, _, _}, r;\n\t}"
               : "=r"(x), "=r"(valid) : "r"(smem_u32(resp)) : "memory");
  return valid ? (long long)(x >> 1) : -1;
}
constexpr int S = 4;
__global__ void __cluster_dims__(2, 1, 1) k(int* count, int* who, int spin) {
  __shared__ __align__(16) uint4 resp[S];
  __shared__ uint64_t full[S], empty[S];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = ctarank();
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1 + 1 + 8); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  cluster_sync();
  int i = 0;
  auto next = [&](bool etx, bool arr) -> long long {
    const int s = i % S; const uint32_t par = (i / S) & 1;
    if (etx) mbar_expect_tx(&full[s], 16);
    mbar_wait(&full[s], par);
    long long t = decode(&resp[s]);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (arr) { if (rank == 0) mbar_arrive(&empty[s]); else arrive_remote(mapa0(&empty[s])); }
    ++i;
    return t;
  };
  auto issue = [&](int j) { const int s = j % S; mbar_wait(&empty[s], ((j / S) & 1) ^ 1); try_cancel(&resp[s], &full[s]); };
  long long t = blockIdx.x >> 1;
  if (warp == 0) {
    if (lane == 0) {
      if (rank == 0) issue(0);
      while (t >= 0) {
        if (rank == 0) { atomicAdd(&count[t], 1); who[t] = blockIdx.x; }
        t = next(true, true);
        if (rank == 0 && t >= 0) issue(i);
      }
    }
  } else if (warp >= 2) {
    while (t >= 0) {
      for (volatile int q = 0; q < spin; ++q) {}
      t = next(false, lane == 0);
      __syncwarp();
    }
  }
  __syncthreads();
  cluster_sync();
}
int main() {
  for (int T : {74, 300, 2048, 20000}) for (int spin : {0, 2000, 50000}) {
    int *count, *who;
    cudaMalloc(&count, T * 4); cudaMalloc(&who, T * 4); cudaMemset(count, 0, T * 4);
    k<<<2 * T, 192>>>(count, who, spin);
    cudaError_t e = cudaDeviceSynchronize();
    int* h = new int[T];
    cudaMemcpy(h, count, T * 4, cudaMemcpyDeviceToHost);
    int bad = 0, zero = 0, multi = 0;
    for (int t = 0; t < T; ++t) { if (h[t] == 0) ++zero; if (h[t] > 1) ++multi; bad += h[t] != 1; }
    printf("T=%d spin=%d err=%s bad=%d (missing %d, duplicated %d)\n", T, spin, cudaGetErrorString(e), bad, zero, multi);
    delete[] h; cudaFree(count); cudaFree(who);
  }
}
