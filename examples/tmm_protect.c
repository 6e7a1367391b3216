/* examples/tmm_protect.c -- the LP hot path driven through the C ABI alone (no Python, no torch):
 * an LP-protected bf16 TMM (Listing 6 shape, L546-554), a simulated crash that leaves one region's
 * stores unpersisted, validation (L183), selective re-execution and re-validation (Listing 7's
 * check-and-recover, L565-578).  Exit status 0 and a final "OK" line on success.
 *
 *   gcc -O2 -Iinclude -I/usr/local/cuda/include examples/tmm_protect.c \
 *       -Lpaper_conf_iiswc_yudhakzs20_b200 -llp -L/usr/local/cuda/lib64 -lcudart \
 *       -Wl,-rpath,'$ORIGIN/../paper_conf_iiswc_yudhakzs20_b200' -o examples/tmm_protect
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "liblp.h"

#define CK(x)                                                                  \
  do {                                                                         \
    lp_status s_ = (x);                                                        \
    if (s_ != LP_OK) {                                                         \
      fprintf(stderr, "%s -> %d: %s\n", #x, (int)s_, lp_last_error());        \
      return 1;                                                                \
    }                                                                          \
  } while (0)
#define CU(x)                                                                  \
  do {                                                                         \
    cudaError_t e_ = (x);                                                      \
    if (e_ != cudaSuccess) {                                                   \
      fprintf(stderr, "%s -> %s\n", #x, cudaGetErrorString(e_));               \
      return 1;                                                                \
    }                                                                          \
  } while (0)

static uint16_t bf16_of_int(int v) { /* small integers are exact in bf16 */
  float f = (float)v;
  uint32_t u;
  memcpy(&u, &f, 4);
  return (uint16_t)(u >> 16);
}

int main(void) {
  const int64_t M = 512, N = 512, K = 256, REG = 128;
  uint16_t* ha = (uint16_t*)malloc(M * K * 2);
  uint16_t* hb = (uint16_t*)malloc(K * N * 2);
  for (int64_t i = 0; i < M * K; ++i) ha[i] = bf16_of_int((int)(i % 5) - 2);  /* integer-valued: exact */
  for (int64_t i = 0; i < K * N; ++i) hb[i] = bf16_of_int((int)(i % 3) - 1);
  void *a, *b, *out, *ck, *ws;
  int64_t *failed, *d_n;
  CU(cudaMalloc(&a, M * K * 2));
  CU(cudaMalloc(&b, K * N * 2));
  CU(cudaMalloc(&out, M * N * 2));
  CU(cudaMemcpy(a, ha, M * K * 2, cudaMemcpyHostToDevice));
  CU(cudaMemcpy(b, hb, K * N * 2, cudaMemcpyHostToDevice));

  lp_config_t cfg;
  memset(&cfg, 0, sizeof cfg);
  cfg.region_m = (int32_t)REG;
  cfg.region_n = (int32_t)REG;
  cfg.cksum = LP_CK_MOD | LP_CK_XOR;      /* the paper's recommendation (L585) */
  cfg.store = LP_STORE_ARRAY;             /* hash-table-less per-region array (L349) */
  lp_handle h;
  CK(lp_config(&cfg, &h));

  lp_workload_t wl;
  memset(&wl, 0, sizeof wl);
  wl.kind = LP_WL_TMM;
  wl.in_dtype = LP_BF16;
  wl.out_dtype = LP_BF16;
  wl.m = M;
  wl.n = N;
  wl.k = K;
  wl.a = a;
  wl.lda = K;
  wl.b = b;
  wl.ldb = N;
  wl.ldc = N;
  wl.row_offset = 0;
  wl.global_m = M;

  int64_t R;
  size_t ck_bytes, ws_bytes;
  CK(lp_num_regions(h, &wl, &R));
  CK(lp_cksum_bytes(h, &wl, &ck_bytes));
  CK(lp_workspace_bytes(h, &wl, &ws_bytes));
  CU(cudaMalloc(&ck, ck_bytes));
  CU(cudaMalloc(&ws, ws_bytes));
  CU(cudaMemset(ws, 0, ws_bytes));          /* zero-filled once (liblp.h) */
  CU(cudaMalloc((void**)&failed, R * 8));
  CU(cudaMalloc((void**)&d_n, 8));

  CK(lp_cksum_init(h, &wl, ck, 0));
  CK(lp_run_protected(h, &wl, out, ck, 0));
  CK(lp_validate(h, &wl, out, ck, failed, R, d_n, ws, 0));
  int64_t n = -1;
  CU(cudaMemcpy(&n, d_n, 8, cudaMemcpyDeviceToHost));
  printf("regions %lld, failed after a clean run: %lld\n", (long long)R, (long long)n);
  if (n != 0) return 1;

  /* golden copy, then a "crash": region (p=2, q=1)'s row 5 never reached memory (stale zeros) */
  uint16_t* gold = (uint16_t*)malloc(M * N * 2);
  CU(cudaMemcpy(gold, out, M * N * 2, cudaMemcpyDeviceToHost));
  const int64_t p = 2, q = 1, rid = p * (N / REG) + q;
  CU(cudaMemset((char*)out + ((p * REG + 5) * N + q * REG) * 2, 0, REG * 2));
  CK(lp_validate(h, &wl, out, ck, failed, R, d_n, ws, 0));
  int64_t f0 = -1;
  CU(cudaMemcpy(&n, d_n, 8, cudaMemcpyDeviceToHost));
  CU(cudaMemcpy(&f0, failed, 8, cudaMemcpyDeviceToHost));
  printf("after the crash: %lld failed region(s), first = %lld (expected %lld)\n", (long long)n, (long long)f0,
         (long long)rid);
  if (n != 1 || f0 != rid) return 1;

  CK(lp_recover(h, &wl, out, ck, failed, d_n, ws, 0));
  CK(lp_validate(h, &wl, out, ck, failed, R, d_n, ws, 0));
  CU(cudaMemcpy(&n, d_n, 8, cudaMemcpyDeviceToHost));
  uint16_t* back = (uint16_t*)malloc(M * N * 2);
  CU(cudaMemcpy(back, out, M * N * 2, cudaMemcpyDeviceToHost));
  const int same = memcmp(back, gold, M * N * 2) == 0;
  printf("after recovery: %lld failed, output %s the golden run\n", (long long)n, same ? "==" : "!=");
  if (n != 0 || !same) return 1;
  CK(lp_destroy(h));
  printf("OK\n");
  return 0;
}
