/*
 * liblp.h -- C ABI of the B200-native Lazy Persistency (LP) hot path.
 *
 * Method: Yudha, Kimura, Zhou, Solihin, "Scalable and Fast Lazy Persistency on
 * GPUs", IISWC 2020.  Citations are PAPER.md line numbers L<n> + section.
 * Readings of passages the paper leaves open are DESIGN.md R1..R20.
 *
 *   lp_config          ~ "#pragma nvm lpcuda_init(tab, nelems, selem)" and the
 *                        checksum type of "lpcuda_checksum(type, tab, key..)"
 *                        (L357, L526-538, §VI)
 *   lp_cksum_init      table initialisation before the protected kernel (L528)
 *   lp_run_protected   the LP region kernel: region body + checksum epilogue +
 *                      lock-free store into the hash-table-less checksum array
 *                      indexed by region id (L181 §IV-A, L192 §IV-B,
 *                      L220-258 Listings 3-4, L349 §V)
 *   lp_validate        recovery-kernel validation: recompute each region's
 *                      checksum from the output, compare with the table,
 *                      compact the failed region ids (L183 §IV-A)
 *   lp_recover         re-execute only the failed regions (idempotent region =
 *                      the original body, L183)
 *
 * Conventions (all calls):
 *  - Every call returns lp_status; nothing throws across the ABI.  On error a
 *    thread-local message is available from lp_last_error().
 *  - Ownership: the caller owns every buffer.  Device buffers (out, cksum,
 *    failed_list, d_n_failed, workspace, rids, stale, records, workload a/b)
 *    are device pointers on cfg.device, allocated by the caller (torch in the
 *    Python binding).  liblp never allocates or frees device memory; the
 *    handle owns only host state.
 *  - Asynchrony: every device-side operation is enqueued on `stream` (a
 *    cudaStream_t passed as void*; NULL = legacy default stream) and the call
 *    returns without synchronising.  Counts live in device memory (int64) so
 *    recovery and NCCL can consume them without a host round trip.
 *  - Argument errors are reported synchronously (LP_ERR_INVALID_ARG) before
 *    anything is enqueued: NULL pointers, M % region_m or N % region_n != 0,
 *    region_n*es % 16 != 0, pointers not 16-byte aligned, failed_cap < R,
 *    unsupported dtype / workload combinations (LP_ERR_UNSUPPORTED), a device
 *    that is not sm_100 (LP_ERR_UNSUPPORTED).  Launch failures return
 *    LP_ERR_CUDA.  Device-side hash-table exhaustion is reported by lp_stats.
 *  - Region ids are GLOBAL: rid = (row_offset/region_m + p) * (n/region_n) + q
 *    for region (p, q) of this shard (Listing 6 keys (blockIdx.x, blockIdx.y),
 *    L553, linearised row-major: Reading R9), so row shards produce disjoint
 *    id ranges.  The array store indexes the caller's table slice with the
 *    LOCAL rid (rid - rid_offset); hash stores key on the global rid.
 */
#ifndef LIBLP_H_
#define LIBLP_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define LP_API __attribute__((visibility("default")))
#else
#define LP_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  LP_OK = 0,
  LP_ERR_INVALID_ARG = 1,
  LP_ERR_UNSUPPORTED = 2,
  LP_ERR_CUDA = 3,
  LP_ERR_CAPACITY = 4,
  LP_ERR_STATE = 5
} lp_status;

/* Checksum types, OR-able (L192: parity = XOR of store values, modular = sum
 * of store values, Adler-32; the paper recommends MOD|XOR, L585).  0 builds
 * the unprotected twin of the same kernel (the overhead denominator). */
typedef enum { LP_CK_NONE = 0u, LP_CK_MOD = 1u, LP_CK_XOR = 2u, LP_CK_ADLER32 = 4u } lp_cksum_bits;

/* Checksum store.  ARRAY is the paper's hash-table-less global array indexed
 * by region id (L349, §V).  QUAD_CAS is the lock-free quadratic-probing table
 * (atomicCAS on the key slot, L267-272); QUAD_LOCK the same table with every
 * insert inside one global spin lock (L81-83, L341 Table III, Reading R15).
 * CUCKOO is the two-table cuckoo table with atomicExch inserts (L269-274;
 * 16-byte entries moved by one 128-bit exchange, Reading R24); CUCKOO_LOCK the
 * same under the global lock.  Hash stores are built for MOD and MOD|XOR. */
typedef enum {
  LP_STORE_ARRAY = 0,
  LP_STORE_QUAD_CAS = 1,
  LP_STORE_QUAD_LOCK = 2,
  LP_STORE_CUCKOO = 3,
  LP_STORE_CUCKOO_LOCK = 4
} lp_store;

/* Element types.  LP_I32 (in = out = int32, wrapping integer multiply-add) is the
 * paper's own TMM type (Listing 2: int *a, *b, *c); SIMT body only. */
typedef enum { LP_F32 = 0, LP_BF16 = 1, LP_I32 = 2 } lp_dtype;

/* Region bodies.  TMM = tiled matrix multiply (Listing 2, Listing 6
 * L546-554), C = A*B, idempotent.  STENCIL5 = 5-point stencil, out-of-place
 * (stand-in for the paper's bandwidth-bound class, Table I; Reading R19).
 * SPMV = CSR sparse matrix x dense vector, y = A*x (the paper's SPMV benchmark,
 * Table I, bandwidth-bound; NEXT row N4): regions are region_n
 * consecutive rows of y (region_m must be 1), i.e. y is viewed as the matrix
 * [m / region_n][region_n] and region p = rows [p*region_n, (p+1)*region_n). */
typedef enum { LP_WL_TMM = 0, LP_WL_STENCIL5 = 1, LP_WL_SPMV = 2 } lp_wl_kind;

/* TMM body implementation: AUTO picks tcgen05 when the shape allows it. */
typedef enum { LP_BODY_AUTO = 0, LP_BODY_SIMT = 1, LP_BODY_TCGEN05 = 2 } lp_body;

/* Crash-injection modes (harness only; the paper has no crash model: Reading R11). */
typedef enum {
  LP_INJ_STALE_WORDS = 0,  /* a seeded run of m in [1, words] words reverts to the stale image */
  LP_INJ_STALE_REGION = 1, /* the whole region reverts to the stale image */
  LP_INJ_BITFLIP = 2,      /* one seeded bit of one seeded word flips */
  LP_INJ_STALE_RECORD = 3  /* the region's record reverts to the sentinel; data intact */
} lp_inject_mode;

typedef void* lp_stream_t; /* cudaStream_t */

typedef struct {
  int32_t region_m, region_n; /* region shape in output elements (L79 granularity trade-off) */
  uint32_t cksum;             /* OR of lp_cksum_bits; 0 = unprotected twin */
  int32_t store;              /* lp_store */
  int32_t device;             /* CUDA device ordinal */
  int32_t body;               /* lp_body */
  uint32_t hash_seed;         /* seed of the hash function for QUAD stores (Reading R14) */
  uint32_t flags;             /* OR of lp_config_flags (A/B switches); 0 = defaults */
} lp_config_t;

/* lp_config_t.flags */
typedef enum {
  LP_FLAG_TC_1CTA = 1u,    /* tcgen05 body: use the 1-SM 128x256 kernel even where the 2-SM CTA-pair kernel applies */
  LP_FLAG_NO_SHUFFLE = 2u, /* SIMT TMM and SPMV bodies: sequential shared-memory reduction instead of warp reduction
                              (the paper's "without parallel reduction" ablation, L343, Table IV) */
  LP_FLAG_NO_FUSED_COMPACT = 8u, /* lp_validate: always compact the failed flags in a separate (PDL) launch instead
                                    of in the last validate CTA for tables of <= 16384 regions (A/B switch) */
  LP_FLAG_NO_PAIRING = 4u, /* tcgen05 bf16 recovery: one 128x128 tile per failed region/tile instead of pairing
                              failed tiles of the same row band into 128x256 tasks (A/B switch) */
  LP_FLAG_RECOVER_TILE128 = 16u, /* tcgen05 bf16 recovery of 32x32 regions: de-duplicate failed regions into 128x128
                                   tiles (paired into 128x256 tasks) instead of 128x64 slices paired into 128x128
                                   tasks (A/B switch; both re-execute every failed region, L51-57) */
  LP_FLAG_CUCKOO_SHORT_CHAINS = 32u, /* cuckoo stores, test hook: the body's inserts give up after 16 evictions
                                       instead of 128, so entries reach the stash and the rehash (L270) runs */
  LP_FLAG_NVLS_COUNT = 64u, /* allow lp_attach_nvls_count: lp_validate all-reduces the failed count through an
                              NVSwitch multicast counter (multimem.red) from the CTA that finalises it */
  LP_FLAG_RECOVER_SLICES128 = 128u, /* tcgen05 bf16 recovery of 128x128 regions: two 128x64 slices per failed region,
                                      grouped 1-4 per task (finer load balance; the two slice partial records are
                                      combined across tasks) instead of same-row pairs of 128x128 tiles (A/B switch) */
  LP_FLAG_TEST_SKIP_REEXEC = 256u /* test hook: lp_recover_revalidate skips the re-execution, so the re-validation
                                     of the failed list must count every listed region */
} lp_config_flags;

typedef struct {
  int32_t kind;      /* lp_wl_kind */
  int32_t in_dtype;  /* lp_dtype of a / b */
  int32_t out_dtype; /* lp_dtype of out */
  int32_t reserved;
  int64_t m, n, k;   /* TMM: out[m,n] = a[m,k] * b[k,n].  STENCIL5: m = rows of this shard, n = W, k unused */
  const void* a;     /* TMM A (row-major, pitch lda elements) / STENCIL5 input (pitch lda) */
  int64_t lda;
  const void* b;     /* TMM B (row-major [k, n], pitch ldb elements); unused for STENCIL5 */
  int64_t ldb;
  int64_t ldc;       /* out row pitch in elements */
  int64_t row_offset, global_m; /* shard: rows [row_offset, row_offset+m) of global_m.
                                   STENCIL5 shards: a points at the input element of global row
                                   row_offset, column 0; the halo rows a - lda (when row_offset > 0) and
                                   a + m*lda (when row_offset + m < global_m) must be readable -- they are
                                   the neighbouring shards' boundary rows, which the caller holds (the
                                   input is read-only, so no exchange happens inside liblp). */
  /* SPMV only (ignored otherwise): m = rows of A (= length of y = out), n = columns
   * (= length of x = b), a = values (f32 [nnz]), b = x (f32 [n]), row_ptr (int64
   * [m + 1], absolute offsets into a / col_idx for this shard's rows), col_idx
   * (int32 [nnz], in [0, n)); ldc, lda, ldb, k are ignored.  Device pointers. */
  const int64_t* row_ptr;
  const int32_t* col_idx;
  int64_t nnz;
} lp_workload_t;

typedef struct lp_ctx* lp_handle;

/* Create a handle for one region shape + checksum type + store. No CUDA call. */
LP_API lp_status lp_config(const lp_config_t* cfg, lp_handle* out);
LP_API lp_status lp_destroy(lp_handle h);

/* R = (m/region_m) * (n/region_n): regions of this shard (L537: nelems = grid.x*grid.y). */
LP_API lp_status lp_num_regions(lp_handle h, const lp_workload_t* wl, int64_t* r);

/* Bytes of the checksum buffer.  ARRAY: R * 4 * selem (selem = popcount(cksum),
 * L528 "number of checksums in an element").  QUAD_*: 64-byte header + cap *
 * 4 * (1 + selem) with cap = smallest prime >= ceil(R / 0.7) (L267 load <= 70%).
 * CUCKOO*: 64-byte header + (2 tables * cap + 256 stash entries) * 16 with
 * cap = smallest prime >= ceil(1.15 R) (total load <= 43.5%, L270).
 * Hash header (u32 words): cap, seed, lock, error, collisions (u64), stash_n,
 * rehashes, max_evict, 7 reserved.  The seed changes when a cuckoo table is
 * rehashed: lookups must read it from the header. */
LP_API lp_status lp_cksum_bytes(lp_handle h, const lp_workload_t* wl, size_t* bytes);

/* Bytes of the scratch `workspace` lp_validate / lp_recover use (flags, scan counters,
 * recovery tile lists, the fused-compaction ticket).  The caller zero-fills it ONCE
 * before its first use (cudaMemset); every call leaves the ticket back at zero, so the
 * workspace can be reused (and replayed in CUDA graphs) without re-initialisation.
 * One workspace per in-flight call (calls sharing a workspace must be stream-ordered). */
LP_API lp_status lp_workspace_bytes(lp_handle h, const lp_workload_t* wl, size_t* bytes);

/* Fill the table with the sentinel 0xFFFFFFFF (Reading R8; hash: all keys empty,
 * collision counter and error flag zero). */
LP_API lp_status lp_cksum_init(lp_handle h, const lp_workload_t* wl, void* cksum, lp_stream_t stream);

/* The LP-protected region kernel: computes out = body(wl) and, in the same
 * kernel, stores one record per region into cksum (no second pass over out).
 * cfg.cksum == 0 runs the unprotected twin (cksum may be NULL).
 * Cuckoo stores: an insert whose eviction walk reaches the bound (a cycle, L270)
 * parks its entry in the table's stash; a one-CTA rehash kernel enqueued after the
 * body (and after lp_recover) then rebuilds T1/T2 in place under a new seed and
 * re-inserts the stash, retrying with further seeds.  It returns at once when the
 * stash is empty.  lp_stats reports error = 1 only if an entry could not be placed. */
LP_API lp_status lp_run_protected(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, lp_stream_t stream);

/* Validation: recompute every region's record from `out`, compare with `cksum`
 * (hash stores: lookup; an absent key counts as failed), write the failed
 * GLOBAL rids in ascending order to failed_list[0 .. *d_n_failed) and the count
 * to *d_n_failed (device int64).  failed_cap must be >= R.  workspace must hold
 * lp_workspace_bytes bytes (zero-filled before first use).  R <= 16384: one launch
 * (the last CTA compacts); larger R: validate + a dependent compaction launch. */
LP_API lp_status lp_validate(lp_handle h, const lp_workload_t* wl, const void* out, const void* cksum, int64_t* failed_list,
                      int64_t failed_cap, int64_t* d_n_failed, void* workspace, lp_stream_t stream);

/* Selective re-execution (eager recovery, L85): re-runs the region body for
 * exactly the regions in failed_list[0 .. *d_n_failed) (global rids of this
 * shard), rewriting their data AND records.  The count is read on the device.
 * `workspace` (optional, lp_workspace_bytes bytes, may be NULL) lets liblp
 * de-duplicate failed regions that share one tensor-core tile (32x32 regions:
 * 16 per 128x128 tile) so each tile is recomputed once; with NULL every listed
 * region recomputes its tile (same final state, more work).  With a workspace and
 * the bf16 tcgen05 body, failed 128x128 tiles of the same 128-row band are also
 * paired into one 128x256 task (A row panel read once for both) when more tiles
 * failed than there are SMs; results are bit-identical either way. */
LP_API lp_status lp_recover(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, const int64_t* failed_list,
                            const int64_t* d_n_failed, void* workspace, lp_stream_t stream);

/* lp_recover that also reports, in *d_n_recovered (device int64; may be NULL), the number of
 * regions whose data and record the recovery kernels rewrote: the entries of the list the kernel
 * consumed times the regions per entry -- *d_n_failed without de-duplication, and (de-duplicated
 * tiles or slices) x (32x32 regions per tile / slice) when several failed 32x32 regions share a
 * tensor-core tile, in which case it can exceed *d_n_failed.  Written on the device after the
 * re-execution kernel, in stream order. */
LP_API lp_status lp_recover_count(lp_handle h, const lp_workload_t* wl, void* out, void* cksum,
                                  const int64_t* failed_list, const int64_t* d_n_failed, void* workspace,
                                  int64_t* d_n_recovered, lp_stream_t stream);

/* Recovery followed by the re-validation of the whole output (steps a10 + a11), with the re-validation split
 * so that most of it overlaps the recovery: the regions the PREVIOUS lp_validate on this workspace did not
 * flag (its per-region flags are read from `workspace`, which must be that call's, untouched since) are
 * re-validated on a liblp-owned side stream while `stream` re-executes the flagged ones (lp_recover_count);
 * after both, the regions of failed_list are re-validated.  Recovery writes only the listed regions' data
 * and array-table records, so the unflagged regions' bytes and records are not written while they are read.
 * *d_n_after (device int64, zeroed by the call) = regions whose record still mismatches (0 after a
 * successful recovery); no failed list is produced (call lp_validate for one if it is not 0).
 * *d_n_recovered as in lp_recover_count (may be NULL).  Work and result equal lp_recover_count +
 * lp_validate; stream-ordered on `stream` (the side stream is forked from and joined back into it with
 * events, so the call may be captured into a CUDA graph; the side stream and events belong to the handle, so
 * concurrent lp_recover_revalidate calls on ONE handle from several host threads are not supported).  Array store with cfg.cksum != 0 only
 * (hash-store inserts can move other keys), and only where the recovery writes exactly the listed regions:
 * the stencil, SpMV, the SIMT TMM and the tcgen05 bf16 TMM with 128x128 regions (the tensor-core bodies
 * with smaller regions rewrite whole recovery tiles); LP_ERR_UNSUPPORTED otherwise.
 * Measured on B200 (bench --split-revalidate): not faster than lp_recover_count + lp_validate for the
 * C2 TMM (0.136 vs 0.128 ms) or the C4 stencil (1.57 vs 1.43 ms) -- the concurrent re-validation contends
 * with the recovery for the L2->SM fabric / DRAM -- so the bench's default path stays sequential. */
LP_API lp_status lp_recover_revalidate(lp_handle h, const lp_workload_t* wl, void* out, void* cksum,
                                       const int64_t* failed_list, const int64_t* d_n_failed, void* workspace,
                                       int64_t* d_n_after, int64_t* d_n_recovered, lp_stream_t stream);

/* The paper's own recovery form (Listing 7; NEXT row N2): ONE kernel
 * with the grid of the original kernel, in which every CTA validates its regions
 * and, if a check fails, re-executes in place (data and record).
 * *d_n_recovered (device int64, zeroed by the call) receives the number of failed
 * (re-executed) regions.  No failed list is produced.
 *  - STENCIL5: one CTA per region.
 *  - TMM (bf16 input, tcgen05 CTA-pair body: m, n % 256 == 0, k % 64 == 0,
 *    128x128 or 32x32 regions): the persistent CTA pairs walk the tile schedule of
 *    lp_run_protected; each CTA first validates its 128-row halves of its pair's
 *    256x256 tiles (all warps, coalesced streaming reads), the pair merges its two
 *    failed-tile bitmasks through distributed shared memory, and the pair's
 *    TMA/MMA/epilogue pipeline then recomputes only the tiles holding a failed
 *    region (every region of such a tile is rewritten with identical bits).
 * Other workloads / bodies: LP_ERR_UNSUPPORTED. */
LP_API lp_status lp_check_recover(lp_handle h, const lp_workload_t* wl, void* out, void* cksum,
                                  int64_t* d_n_recovered, lp_stream_t stream);

/* lp_check_recover with a workspace (lp_workspace_bytes bytes; NULL = the static form above).  TMM: the
 * balanced form -- a cooperative launch (at most the co-resident CTA pairs) whose CTAs publish their
 * failed tiles to a global bitmask in the workspace and pass a grid barrier after the check phase; the
 * j-th failed tile then goes to pair j % npairs, so the recompute spreads over every pair instead of
 * staying on the pairs that own the failed tiles.  Same final state and count.  STENCIL5: as
 * lp_check_recover. */
LP_API lp_status lp_check_recover_ws(lp_handle h, const lp_workload_t* wl, void* out, void* cksum,
                                     int64_t* d_n_recovered, void* workspace, lp_stream_t stream);

/* NVLS-fused failed-count all-reduce (needs cfg.flags & LP_FLAG_NVLS_COUNT).
 * mc_counter = the multicast (NVLS) address and uc_counter = this rank's unicast address of the same
 * 64-byte-aligned, >= 64-byte counter buffer, bound to a multicast object on every one of the
 * world_size ranks and zero-filled on all of them before the first lp_validate (e.g. torch symmetric
 * memory: rendezvous(...).multicast_ptr / buffer_ptrs[rank]).  Afterwards every lp_validate on this
 * handle ends with the CTA that writes *d_n_failed adding the shard's count with
 * multimem.red.add.u64 into every rank's copy, signalling its arrival the same way and waiting for all
 * ranks of this epoch; ((uint64_t*)uc_counter)[4] then holds the all-rank failed count (the local list
 * and *d_n_failed are unchanged).  Every rank must call lp_validate the same number of times.
 * mc_counter == uc_counter with world_size == 1 is a single-GPU emulation (plain atomics) that
 * exercises the epoch logic; NULL, NULL detaches.  The multimem path itself needs >= 2 GPUs on an
 * NVSwitch fabric: a 1-device multicast object cannot be created (cuMulticastCreate -> invalid value). */
LP_API lp_status lp_attach_nvls_count(lp_handle h, void* mc_counter, void* uc_counter, int32_t world_size);

/* Records of every region of `out` (uint32 [R][selem], order MOD, XOR, ADLER)
 * without comparing -- for parity tests against the oracle. */
LP_API lp_status lp_region_checksums(lp_handle h, const lp_workload_t* wl, const void* out, uint32_t* records,
                              lp_stream_t stream);

/* Crash injection (harness only): corrupt the n regions whose GLOBAL rids are
 * in device array rids[0..n) (ids outside this shard's range are skipped)
 * according to `mode` (lp_inject_mode), using the
 * stale image `stale` (same shape/pitch as out; may be NULL for BITFLIP and
 * STALE_RECORD) and counter-based choices seeded by `seed`. */
LP_API lp_status lp_inject(lp_handle h, const lp_workload_t* wl, void* out, void* cksum, const void* stale,
                    const int64_t* rids, int64_t n, uint32_t mode, uint64_t seed, lp_stream_t stream);

/* Hash-store statistics: d_stats (device int64[2]) <- {collisions (sum over
 * inserts of probes-1), error flag (1 = a probe sequence was exhausted)}.
 * ARRAY store: {0, 0}. */
LP_API lp_status lp_stats(lp_handle h, const lp_workload_t* wl, const void* cksum, int64_t* d_stats, lp_stream_t stream);

/* False-negative study (NEXT row N3, L53/L192 "random error injection"): run `trials`
 * seeded corruption trials of a region of `region_words` 32-bit words under
 * `model` (0 random words, 1 bit flips, 2 adversarial same-bit pair, 3 zeroed
 * words; k in [1, kmax] corruptions, kmax <= 8) and count, in device
 * d_counts (uint64[7]): {trials that changed the region, undetected by MOD, XOR,
 * MOD|XOR, ADLER32, MOD|XOR|ADLER32, no-op trials}.  The first dump_trials trials
 * are written to device dump (uint32[dump_trials][26]: k, positions[8], old
 * words[8], new words[8], detected bits MOD=1 XOR=2 ADLER=4, changed=8) for
 * re-checking against the CPU oracle; dump may be NULL. */
LP_API lp_status lp_fn_study(lp_handle h, uint32_t model, int32_t kmax, int64_t region_words, uint64_t seed,
                             int64_t trials, uint64_t* d_counts, uint32_t* dump, int64_t dump_trials,
                             lp_stream_t stream);

/* Number of SMs / cached device properties are queried lazily; this returns
 * the device's SM count (0 if no device). */
LP_API int32_t lp_device_sm_count(lp_handle h);

/* Thread-local text of the last error ("" if none). */
LP_API const char* lp_last_error(void);

/* ABI version (major*100 + minor). */
LP_API int32_t lp_abi_version(void);

#ifdef __cplusplus
}
#endif

#endif /* LIBLP_H_ */
