/*
 * oracle/lp_oracle.c -- plain, slow, obviously-correct CPU oracle for the
 * Lazy Persistency (LP) hot path of Yudha et al., "Scalable and Fast Lazy
 * Persistency on GPUs" (IISWC 2020).  Citations are PAPER.md line numbers
 * (L<n>) with the section / listing they belong to.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_iiswc_yudhakzs20_b200/csrc); neither side includes the other.
 *
 * Single-threaded, no blocking, no reordering beyond the definitions below.
 * Pins (tests/test_oracle_pins.py) tie every function to something other than
 * itself: paper worked examples, zlib, brute force, closed forms.
 *
 * Readings of the paper used here are DESIGN.md R1..R18 (= SURVEY.md §8c c1..c18).
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -shared -fPIC
 */
#include <stdint.h>
#include <string.h>

#define LPO_MOD   1u   /* modular checksum: store values added       (L192, §IV-B) */
#define LPO_XOR   2u   /* parity checksum:  store values XORed       (L192, §IV-B) */
#define LPO_ADLER 4u   /* Adler-32 [24],[25] as in zlib              (L192, §IV-B) */
#define ADLER_BASE 65521u

/* ------------------------------------------------------------------------ */
/* Float -> "ordered integer" (L260-261, Fig. 2): the concatenation of sign,  */
/* exponent and mantissa bits, i.e. the raw IEEE-754 bit pattern.  Worked     */
/* example in the paper: 3.5f -> 1080033280.  (Reading R2.)                   */
uint32_t lpo_float_word(float v) {
  uint32_t w;
  memcpy(&w, &v, 4);
  return w;
}

/* ------------------------------------------------------------------------ */
/* Adler-32, textbook sequential definition (zlib; L192 "Adler-32 [24],[25]"): */
/*   A = 1 + sum d_i (mod 65521); B = sum over i of A_i (mod 65521).          */
uint32_t lpo_adler32(const uint8_t* buf, int64_t n) {
  uint32_t a = 1, b = 0;
  for (int64_t i = 0; i < n; ++i) {
    a = (a + buf[i]) % ADLER_BASE;
    b = (b + a) % ADLER_BASE;
  }
  return (b << 16) | a;
}

static int popcount3(uint32_t m) { return (int)((m & 1u) + ((m >> 1) & 1u) + ((m >> 2) & 1u)); }

int lpo_selem(uint32_t mask) { return popcount3(mask & 7u); }

/* ------------------------------------------------------------------------ */
/* Region record (L192: "the checksum is computed over all store values that  */
/* must persist in an LP region"; L349: one checksum entry per region).       */
/* Region (p,q) of an output with row pitch ldc elements of es bytes:         */
/* word stream = for i in [0,RM) ascending, for j in [0, RN*es/4) ascending,  */
/* the little-endian u32 at byte ((p*RM+i)*ldc + q*RN)*es + 4j (Reading R1,   */
/* R6: fp32 -> its IEEE bits; bf16 -> two elements per word, even column in   */
/* the low half, i.e. the memory image).  MOD = sum w mod 2^32, XOR = xor w,  */
/* ADLER = adler32 of the same bytes in address order (Reading R5).           */
/* The record is [MOD?, XOR?, ADLER?] in that order (Reading R7).             */
void lpo_region_record(const void* out, int64_t ldc, int es, int64_t p, int64_t q, int RM, int RN,
                       uint32_t mask, uint32_t* rec) {
  const uint8_t* base = (const uint8_t*)out;
  const int64_t row_bytes = (int64_t)RN * es;
  const int64_t words = row_bytes / 4;
  uint32_t mod = 0, xr = 0, a = 1, b = 0;
  for (int64_t i = 0; i < RM; ++i) {
    const uint8_t* row = base + ((p * RM + i) * ldc + q * (int64_t)RN) * es;
    for (int64_t j = 0; j < words; ++j) {
      uint32_t w;
      memcpy(&w, row + 4 * j, 4);
      mod += w;                 /* wraps mod 2^32 (Reading R1) */
      xr ^= w;
    }
    if (mask & LPO_ADLER) {
      for (int64_t t = 0; t < row_bytes; ++t) {  /* sequential zlib loop over the row's bytes */
        a = (a + row[t]) % ADLER_BASE;
        b = (b + a) % ADLER_BASE;
      }
    }
  }
  int k = 0;
  if (mask & LPO_MOD) rec[k++] = mod;
  if (mask & LPO_XOR) rec[k++] = xr;
  if (mask & LPO_ADLER) rec[k++] = (b << 16) | a;
}

/* All records of an M x N output, rid = p*(N/RN) + q (Listing 6 keys         */
/* (blockIdx.x, blockIdx.y), L553, linearised row-major: Reading R9).         */
void lpo_records(const void* out, int64_t M, int64_t N, int64_t ldc, int es, int RM, int RN, uint32_t mask,
                 uint32_t* recs) {
  const int selem = lpo_selem(mask);
  const int64_t P = M / RM, Q = N / RN;
  for (int64_t p = 0; p < P; ++p)
    for (int64_t q = 0; q < Q; ++q) lpo_region_record(out, ldc, es, p, q, RM, RN, mask, recs + (p * Q + q) * selem);
}

/* ------------------------------------------------------------------------ */
/* Validation (L183, §IV-A: "first validates the checksum for each thread     */
/* block by fetching the corresponding data from memory, computing their      */
/* checksums, and then comparing them with the ones stored in the checksum    */
/* table").  Array store (L349): table entry for rid is table[rid*selem ..].  */
/* Output: ascending global rids (rid + rid_offset) whose recomputed record   */
/* differs in any word (Reading R12).  Returns the count.                     */
int64_t lpo_validate_array(const void* out, const uint32_t* table, int64_t M, int64_t N, int64_t ldc, int es,
                           int RM, int RN, uint32_t mask, int64_t rid_offset, int64_t* failed) {
  const int selem = lpo_selem(mask);
  const int64_t P = M / RM, Q = N / RN;
  int64_t nf = 0;
  uint32_t rec[3];
  for (int64_t p = 0; p < P; ++p)
    for (int64_t q = 0; q < Q; ++q) {
      const int64_t rid = p * Q + q;
      lpo_region_record(out, ldc, es, p, q, RM, RN, mask, rec);
      int bad = 0;
      for (int s = 0; s < selem; ++s) bad |= (rec[s] != table[rid * selem + s]);
      if (bad) failed[nf++] = rid + rid_offset;
    }
  return nf;
}

/* ------------------------------------------------------------------------ */
/* Quadratic-probing hash table (L267, §IV-C: "adding i^2 to the original     */
/* index in the i-th iteration"; open addressing only, L265).  Hash function  */
/* is unstated: Reading R14 = murmur3 fmix32(rid ^ seed) mod cap.            */
/* Entry layout: u32 key (0xFFFFFFFF = empty) followed by selem record words. */
uint32_t lpo_quad_hash(uint32_t key, uint32_t seed, uint32_t cap) {
  uint32_t h = key ^ seed;
  h ^= h >> 16;
  h *= 0x85ebca6bu;
  h ^= h >> 13;
  h *= 0xc2b2ae35u;
  h ^= h >> 16;
  return h % cap;
}

/* slot visited at probe i (i = 0 is the home slot) */
uint32_t lpo_quad_probe(uint32_t key, uint32_t seed, uint32_t cap, uint32_t i) {
  uint64_t s = (uint64_t)lpo_quad_hash(key, seed, cap) + (uint64_t)i * (uint64_t)i;
  return (uint32_t)(s % cap);
}

/* Lookup (L270: "lookups are not in the critical path"): walk the probe      */
/* sequence until the key or an empty slot. Returns 1 and the record if found.*/
int lpo_quad_lookup(const uint32_t* table, uint32_t cap, int selem, uint32_t key, uint32_t seed, uint32_t* rec) {
  for (uint32_t i = 0; i < cap; ++i) {
    const uint32_t* e = table + (uint64_t)lpo_quad_probe(key, seed, cap, i) * (uint64_t)(1 + selem);
    if (e[0] == key) {
      for (int s = 0; s < selem; ++s) rec[s] = e[1 + s];
      return 1;
    }
    if (e[0] == 0xFFFFFFFFu) return 0;
  }
  return 0;
}

/* Sequential insert of key with record into the table (reference semantics  */
/* of one insertion; returns the number of probes used, 0 if the table is     */
/* exhausted).  Used by the pins of the probe order (L267's +1, +4, +9).      */
uint32_t lpo_quad_insert(uint32_t* table, uint32_t cap, int selem, uint32_t key, uint32_t seed, const uint32_t* rec) {
  for (uint32_t i = 0; i < cap; ++i) {
    uint32_t* e = table + (uint64_t)lpo_quad_probe(key, seed, cap, i) * (uint64_t)(1 + selem);
    if (e[0] == 0xFFFFFFFFu || e[0] == key) {
      e[0] = key;
      for (int s = 0; s < selem; ++s) e[1 + s] = rec[s];
      return i + 1;
    }
  }
  return 0;
}

/* Validation against a hash store: a key that is absent counts as failed     */
/* (Reading R12; L183 validation, L270 lookup).                               */
int64_t lpo_validate_quad(const void* out, const uint32_t* table, uint32_t cap, uint32_t seed, int64_t M, int64_t N,
                          int64_t ldc, int es, int RM, int RN, uint32_t mask, int64_t rid_offset, int64_t* failed) {
  const int selem = lpo_selem(mask);
  const int64_t P = M / RM, Q = N / RN;
  int64_t nf = 0;
  uint32_t rec[3], stored[3];
  for (int64_t p = 0; p < P; ++p)
    for (int64_t q = 0; q < Q; ++q) {
      const int64_t rid = p * Q + q + rid_offset;
      lpo_region_record(out, ldc, es, p, q, RM, RN, mask, rec);
      int bad = !lpo_quad_lookup(table, cap, selem, (uint32_t)rid, seed, stored);
      for (int s = 0; !bad && s < selem; ++s) bad |= (rec[s] != stored[s]);
      if (bad) failed[nf++] = rid;
    }
  return nf;
}

/* ------------------------------------------------------------------------ */
/* Cuckoo hashing (L269-270, Fig. 4): tables T1, T2 with hash functions H1, H2. */
/* Insert puts the key at T1[H1(k)]; an occupant is evicted to the other table */
/* (T2[H2(.)], then T1[H1(.)], ...); L270 "The lookup process ... find all    */
/* possible indices pointed by all hashing functions".  Hash functions are     */
/* unstated: Reading R24 = H1 = fmix32(k ^ seed) mod cap, H2 = fmix32(k ^      */
/* (seed * 0x9E3779B9 + 0x7F4A7C15)) mod cap.  Entry = 4 u32: key, 3 record    */
/* words (unused words 0).  Table t starts at entry t * cap.                  */
uint32_t lpo_cuckoo_hash(int t, uint32_t key, uint32_t seed, uint32_t cap) {
  return t == 0 ? lpo_quad_hash(key, seed, cap) : lpo_quad_hash(key, seed * 0x9E3779B9u + 0x7F4A7C15u, cap);
}

int lpo_cuckoo_lookup(const uint32_t* tab, uint32_t cap, int selem, uint32_t key, uint32_t seed, uint32_t* rec) {
  for (int t = 0; t < 2; ++t) {
    const uint32_t* e = tab + 4 * ((uint64_t)t * cap + lpo_cuckoo_hash(t, key, seed, cap));
    if (e[0] == key) {
      for (int s = 0; s < selem; ++s) rec[s] = e[1 + s];
      return 1;
    }
  }
  return 0;
}

/* Sequential insert; returns the number of placements (1 = no eviction), 0 if */
/* the chain exceeds max_evict (the paper would rehash).                       */
uint32_t lpo_cuckoo_insert(uint32_t* tab, uint32_t cap, int selem, uint32_t key, uint32_t seed, const uint32_t* rec,
                           int max_evict) {
  uint32_t e[4] = {key, 0, 0, 0};
  for (int s = 0; s < selem; ++s) e[1 + s] = rec[s];
  for (int t2 = 0; t2 < 2; ++t2) { /* an existing key is updated in place (re-insertion on recovery) */
    uint32_t* slot = tab + 4 * ((uint64_t)t2 * cap + lpo_cuckoo_hash(t2, key, seed, cap));
    if (slot[0] == key) {
      memcpy(slot, e, 16);
      return 1;
    }
  }
  int t = 0;
  for (int i = 0; i < max_evict; ++i) {
    uint32_t* slot = tab + 4 * ((uint64_t)t * cap + lpo_cuckoo_hash(t, e[0], seed, cap));
    uint32_t old[4];
    memcpy(old, slot, 16);
    memcpy(slot, e, 16);
    if (old[0] == 0xFFFFFFFFu || old[0] == e[0]) return (uint32_t)i + 1;
    memcpy(e, old, 16);
    t ^= 1;
  }
  return 0;
}

int64_t lpo_validate_cuckoo(const void* out, const uint32_t* tab, uint32_t cap, uint32_t seed, int64_t M, int64_t N,
                            int64_t ldc, int es, int RM, int RN, uint32_t mask, int64_t rid_offset, int64_t* failed) {
  const int selem = lpo_selem(mask);
  const int64_t P = M / RM, Q = N / RN;
  int64_t nf = 0;
  uint32_t rec[3], stored[3];
  for (int64_t p = 0; p < P; ++p)
    for (int64_t q = 0; q < Q; ++q) {
      const int64_t rid = p * Q + q + rid_offset;
      lpo_region_record(out, ldc, es, p, q, RM, RN, mask, rec);
      int bad = !lpo_cuckoo_lookup(tab, cap, selem, (uint32_t)rid, seed, stored);
      for (int s = 0; !bad && s < selem; ++s) bad |= (rec[s] != stored[s]);
      if (bad) failed[nf++] = rid;
    }
  return nf;
}

/* ------------------------------------------------------------------------ */
/* Region body 1: tiled matrix multiply (Listing 2, Listing 6        */
/* L546-554): C = A * B, A [M x K] row-major, B [K x N] row-major.  Plain     */
/* triple loop in fp64 for the RM x RN block at (row0, col0).  is_bf16 selects */
/* the operand storage: 0 fp32, 1 bf16 bits (widened exactly), 2 int32 (exact */
/* while |partial sums| < 2^53).                                              */
/* operand element as fp64: dtype 0 = fp32, 1 = bf16 bits, 2 = int32 (Listing 2's int TMM) */
static double load_elem(const void* base, int is_bf16, int64_t idx) {
  if (is_bf16 == 2) {
    int32_t v;
    memcpy(&v, (const uint8_t*)base + 4 * idx, 4);
    return (double)v;
  }
  if (is_bf16) {
    uint16_t h;
    memcpy(&h, (const uint8_t*)base + 2 * idx, 2);
    uint32_t w = (uint32_t)h << 16;
    float f;
    memcpy(&f, &w, 4);
    return (double)f;
  }
  float f;
  memcpy(&f, (const uint8_t*)base + 4 * idx, 4);
  return (double)f;
}

void lpo_gemm_block_f64(const void* A, int64_t lda, const void* B, int64_t ldb, int is_bf16, int64_t K,
                        int64_t row0, int64_t col0, int64_t rows, int64_t cols, double* C /* rows x cols */) {
  for (int64_t i = 0; i < rows; ++i)
    for (int64_t j = 0; j < cols; ++j) {
      double s = 0.0;
      for (int64_t k = 0; k < K; ++k)
        s += load_elem(A, is_bf16, (row0 + i) * lda + k) * load_elem(B, is_bf16, k * ldb + col0 + j);
      C[i * cols + j] = s;
    }
}

/* fp64 -> fp32 (round to nearest) -> bf16 round-to-nearest-even, as bits.    */
/* Used for integer-valued inputs, whose fp64 block is exact (Reading R18).   */
void lpo_round_bf16(const double* x, int64_t n, uint16_t* out) {
  for (int64_t i = 0; i < n; ++i) {
    float f = (float)x[i];
    uint32_t u;
    memcpy(&u, &f, 4);
    uint32_t lsb = (u >> 16) & 1u;
    u += 0x7FFFu + lsb;
    out[i] = (uint16_t)(u >> 16);
  }
}

/* ------------------------------------------------------------------------ */
/* Region body 2: 5-point stencil (stand-in for the paper's bandwidth-bound   */
/* class, Table I; Reading R19).  fp32, zero outside the domain:     */
/*   out[i][j] = 0.5*in[i][j] + 0.125*(((in[i-1][j] + in[i+1][j])            */
/*                                      + in[i][j-1]) + in[i][j+1])           */
/* in exactly that order, every operation rounded to fp32 (no contraction).   */
static float at(const float* in, int64_t H, int64_t W, int64_t ld, int64_t i, int64_t j) {
  if (i < 0 || i >= H || j < 0 || j >= W) return 0.0f;
  return in[i * ld + j];
}

void lpo_stencil5_block(const float* in, int64_t H, int64_t W, int64_t ld, int64_t row0, int64_t col0, int64_t rows,
                        int64_t cols, float* out /* rows x cols */) {
  for (int64_t i = row0; i < row0 + rows; ++i)
    for (int64_t j = col0; j < col0 + cols; ++j) {
      volatile float ud = at(in, H, W, ld, i - 1, j) + at(in, H, W, ld, i + 1, j);
      volatile float udl = ud + at(in, H, W, ld, i, j - 1);
      volatile float s = udl + at(in, H, W, ld, i, j + 1);
      volatile float c = 0.5f * at(in, H, W, ld, i, j);
      volatile float t = 0.125f * s;
      out[(i - row0) * cols + (j - col0)] = c + t;
    }
}

/* ------------------------------------------------------------------------ */
/* Region body 3: sparse matrix - dense vector product, CSR (the paper's SPMV */
/* benchmark, Table I, bandwidth-bound; NEXT row N4).  Definition:   */
/*   y[i] = sum_{k = row_ptr[i]}^{row_ptr[i+1]-1} val[k] * x[col[k]]          */
/* summed in fp64 in CSR order (exact for integer-valued inputs; the GPU's    */
/* fp32 result is compared within the stated tolerance otherwise).            */
/* Rows [row0, row0+rows) of the matrix; row_ptr holds absolute offsets.      */
void lpo_spmv_rows(const int64_t* row_ptr, const int32_t* col, const float* val, const float* x, int64_t row0,
                   int64_t rows, double* y /* rows */) {
  for (int64_t i = 0; i < rows; ++i) {
    double s = 0.0;
    for (int64_t k = row_ptr[row0 + i]; k < row_ptr[row0 + i + 1]; ++k) s += (double)val[k] * (double)x[col[k]];
    y[i] = s;
  }
}
