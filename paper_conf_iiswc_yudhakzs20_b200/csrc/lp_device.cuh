// lp_device.cuh -- device-side LP building blocks shared by every CUDA kernel of liblp.
//
//  * per-thread checksum partials over the exact 32-bit words a kernel stores
//    (L192 §IV-B: parity = XOR, modular = sum, Adler-32; L260-261 Fig. 2: the
//    float's raw bits are the word -- Readings R1, R2, R5, R6);
//  * warp reduction with one redux.sync per checksum (the B200 form of
//    Listing 4's shfl_down ladder, L244-258) and the block combine through a
//    small shared array (Listing 3);
//  * the lock-free record store into the hash-table-less array (L349 §V) and
//    the hash-store ablation (L265-274, L341).
//
// Adler-32 uses the order-free closed form so the partials can be reduced in
// any order: for region bytes d_1..d_n,
//   A = (1 + S) mod 65521,  B = (n + (n+1) S - W) mod 65521,
//   S = sum d_i,  W = sum i*d_i.
// Each 32-bit word at 1-based byte position p contributes S += dp4a(w, 1111),
// W += p*dp4a(w,1111) + dp4a(w, 0x03020100).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace lp {

constexpr uint32_t kMod = 1u, kXor = 2u, kAdler = 4u;
constexpr uint32_t kAdlerBase = 65521u;
constexpr uint32_t kSentinel = 0xFFFFFFFFu;
constexpr uint32_t kEmptyKey = 0xFFFFFFFFu;

__host__ __device__ constexpr int selem_of(uint32_t mask) {
  return (int)((mask & 1u) + ((mask >> 1) & 1u) + ((mask >> 2) & 1u));
}

// Per-thread partials.  MASK is a compile-time checksum set so the unprotected
// twin (MASK = 0) compiles to exactly the body.
template <uint32_t MASK>
struct CkPartial {
  uint32_t mod = 0, xr = 0, s = 0;
  uint64_t w = 0;

  // word: the stored 32-bit pattern; pos: 1-based byte position of its first
  // byte inside the region's byte stream (only used by Adler).
  __device__ __forceinline__ void add(uint32_t word, uint32_t pos) {
    if constexpr ((MASK & kMod) != 0) mod += word;
    if constexpr ((MASK & kXor) != 0) xr ^= word;
    if constexpr ((MASK & kAdler) != 0) {
      const uint32_t bs = (uint32_t)__dp4a(word, 0x01010101u, 0u);
      const uint32_t ws = (uint32_t)__dp4a(word, 0x03020100u, 0u);
      s += bs;
      w += (uint64_t)pos * bs + ws;
    }
  }
  // four consecutive words (byte positions pos, pos + 4, pos + 8, pos + 12): the same sums as four
  // add() calls, with Adler's position weights folded per 16 bytes -- sum_k (pos + 4k) * bs_k + ws_k
  // = pos * sum_k bs_k + sum_k dp4a(word_k, {4k, 4k+1, 4k+2, 4k+3}) -- so one 64-bit multiply-add
  // per vector instead of four.
  __device__ __forceinline__ void add4(uint32_t x, uint32_t y, uint32_t z, uint32_t v, uint32_t pos) {
    if constexpr ((MASK & kMod) != 0) mod += (x + y) + (z + v);
    if constexpr ((MASK & kXor) != 0) xr ^= x ^ y ^ z ^ v;
    if constexpr ((MASK & kAdler) != 0) {
      const uint32_t bs = (uint32_t)__dp4a(x, 0x01010101u, __dp4a(y, 0x01010101u,
                                           __dp4a(z, 0x01010101u, __dp4a(v, 0x01010101u, 0u))));
      const uint32_t ws = (uint32_t)__dp4a(x, 0x03020100u, __dp4a(y, 0x07060504u,
                                           __dp4a(z, 0x0B0A0908u, __dp4a(v, 0x0F0E0D0Cu, 0u))));
      s += bs;
      w += (uint64_t)pos * bs + ws;
    }
  }
  __device__ __forceinline__ void merge(const CkPartial& o) {
    mod += o.mod;
    xr ^= o.xr;
    s += o.s;
    w += o.w;
  }
};

// Reduced record of one region (the value every lane holds after warp_reduce).
struct CkRecord {
  uint32_t mod, xr, s, wmod;  // s = byte sum (exact), wmod = W mod 65521
};

template <uint32_t MASK>
__device__ __forceinline__ CkRecord warp_reduce(const CkPartial<MASK>& p, uint32_t lanes = 0xFFFFFFFFu) {
  CkRecord r{0u, 0u, 0u, 0u};
  if constexpr ((MASK & kMod) != 0) r.mod = __reduce_add_sync(lanes, p.mod);
  if constexpr ((MASK & kXor) != 0) r.xr = __reduce_xor_sync(lanes, p.xr);
  if constexpr ((MASK & kAdler) != 0) {
    r.s = __reduce_add_sync(lanes, p.s);
    r.wmod = __reduce_add_sync(lanes, (uint32_t)(p.w % kAdlerBase));
  }
  return r;
}

// Reduction over aligned groups of 2^lg_log2 lanes (every lane of a group ends with its group's record).
template <uint32_t MASK>
__device__ __forceinline__ CkRecord segment_reduce(const CkPartial<MASK>& p, int lg_log2) {
  if (lg_log2 == 5) return warp_reduce<MASK>(p);
  CkRecord r{p.mod, p.xr, p.s, 0u};
  if constexpr ((MASK & kAdler) != 0) r.wmod = (uint32_t)(p.w % kAdlerBase);
  for (int o = (1 << lg_log2) >> 1; o > 0; o >>= 1) {
    if constexpr ((MASK & kMod) != 0) r.mod += __shfl_xor_sync(0xFFFFFFFFu, r.mod, o);
    if constexpr ((MASK & kXor) != 0) r.xr ^= __shfl_xor_sync(0xFFFFFFFFu, r.xr, o);
    if constexpr ((MASK & kAdler) != 0) {
      r.s += __shfl_xor_sync(0xFFFFFFFFu, r.s, o);
      r.wmod += __shfl_xor_sync(0xFFFFFFFFu, r.wmod, o);
    }
  }
  return r;
}

__device__ __forceinline__ CkRecord combine(CkRecord a, const CkRecord& b) {
  a.mod += b.mod;
  a.xr ^= b.xr;
  a.s += b.s;
  a.wmod = (a.wmod % kAdlerBase) + (b.wmod % kAdlerBase);
  return a;
}

// Final Adler-32 value of a region of nbytes bytes from (S, W mod 65521).
__device__ __forceinline__ uint32_t adler_finish(uint32_t s, uint32_t wmod, uint64_t nbytes) {
  const uint64_t P = kAdlerBase;
  const uint64_t a = (1ull + s) % P;
  const uint64_t n = nbytes % P, n1 = (nbytes + 1) % P;
  const uint64_t b = (n + (n1 * (s % P)) % P + P - (wmod % P)) % P;
  return (uint32_t)((b << 16) | a);
}

// Record words in the fixed order MOD, XOR, ADLER (Reading R7).
template <uint32_t MASK>
__device__ __forceinline__ int record_words(const CkRecord& r, uint64_t nbytes, uint32_t* out3) {
  int k = 0;
  if constexpr ((MASK & kMod) != 0) out3[k++] = r.mod;
  if constexpr ((MASK & kXor) != 0) out3[k++] = r.xr;
  if constexpr ((MASK & kAdler) != 0) out3[k++] = adler_finish(r.s, r.wmod, nbytes);
  return k;
}

// ---------------------------------------------------------------------------
// Stores.  Array store (L349): one plain store per region into
// table[local_rid * selem], no atomics and no fences (lazy persist, L55).
template <uint32_t MASK>
__device__ __forceinline__ void store_array(uint32_t* table, int64_t local_rid, const uint32_t* w) {
  constexpr int S = selem_of(MASK);
  uint32_t* dst = table + local_rid * S;
  if constexpr (S == 1) {
    dst[0] = w[0];
  } else if constexpr (S == 2) {
    if ((((uintptr_t)dst) & 7u) == 0) {
      *reinterpret_cast<uint2*>(dst) = make_uint2(w[0], w[1]);
    } else {
      dst[0] = w[0];
      dst[1] = w[1];
    }
  } else if constexpr (S == 3) {
    dst[0] = w[0];
    dst[1] = w[1];
    dst[2] = w[2];
  }
}

// Hash-store layout inside the caller's cksum buffer (Reading R14):
//   [0]  u32 cap      [1] u32 seed     [2] u32 lock word   [3] u32 error flag
//   [4..5] u64 collisions (sum of probes-1)
//   [6]  u32 stash_n (cuckoo: entries parked by chains that hit the eviction bound)
//   [7]  u32 rehashes (cuckoo: completed rehash attempts)  [8] u32 max_evict (0 = kCuckooMaxEvict)
//   [9..15] reserved
//   then cap entries of (1 + selem) u32: key (0xFFFFFFFF = empty), record   (quadratic probing)
//   or   T1[cap], T2[cap] 16-byte entries + a stash of kCuckooStash entries (cuckoo).
struct HashHeader {
  uint32_t cap, seed, lock, error;
  unsigned long long collisions;
  uint32_t stash_n, rehashes, max_evict;
  uint32_t reserved[7];
};
static_assert(sizeof(HashHeader) == 64, "hash header is 64 bytes");

__host__ __device__ __forceinline__ uint32_t hash_fmix32(uint32_t key, uint32_t seed) {
  uint32_t h = key ^ seed;
  h ^= h >> 16;
  h *= 0x85ebca6bu;
  h ^= h >> 13;
  h *= 0xc2b2ae35u;
  h ^= h >> 16;
  return h;
}

// Lock-free insert (L272: atomicCAS on the key slot makes sure the entry is
// empty before inserting; probe i visits home + i^2, L267).  Called by ONE
// thread per region.  Returns the number of probes.
template <uint32_t MASK>
__device__ __forceinline__ uint32_t quad_insert(uint32_t* ckbuf, uint32_t rid, const uint32_t* w) {
  constexpr int S = selem_of(MASK);
  HashHeader* hdr = reinterpret_cast<HashHeader*>(ckbuf);
  uint32_t* ent = ckbuf + sizeof(HashHeader) / 4;
  const uint32_t cap = hdr->cap;
  const uint32_t home = hash_fmix32(rid, hdr->seed) % cap;
  for (uint32_t i = 0; i < cap; ++i) {
    const uint32_t slot = (uint32_t)(((uint64_t)home + (uint64_t)i * i) % cap);
    uint32_t* e = ent + (uint64_t)slot * (1 + S);
    const uint32_t prev = atomicCAS(e, kEmptyKey, rid);
    if (prev == kEmptyKey || prev == rid) {
#pragma unroll
      for (int s = 0; s < S; ++s) e[1 + s] = w[s];
      if (i) atomicAdd(&hdr->collisions, (unsigned long long)i);
      return i + 1;
    }
  }
  atomicExch(&hdr->error, 1u);
  return 0;
}

// Lock-based variant (L81-83 CPU style; L341 "lock-based"): the whole probe +
// insert runs inside one global spin lock (Reading R15).
template <uint32_t MASK>
__device__ __forceinline__ uint32_t quad_insert_locked(uint32_t* ckbuf, uint32_t rid, const uint32_t* w) {
  constexpr int S = selem_of(MASK);
  HashHeader* hdr = reinterpret_cast<HashHeader*>(ckbuf);
  uint32_t* ent = ckbuf + sizeof(HashHeader) / 4;
  while (atomicCAS(&hdr->lock, 0u, 1u) != 0u) {
    __nanosleep(32);
  }
  __threadfence();
  const uint32_t cap = *((volatile uint32_t*)&hdr->cap);
  const uint32_t home = hash_fmix32(rid, hdr->seed) % cap;
  uint32_t probes = 0;
  for (uint32_t i = 0; i < cap; ++i) {
    const uint32_t slot = (uint32_t)(((uint64_t)home + (uint64_t)i * i) % cap);
    volatile uint32_t* e = ent + (uint64_t)slot * (1 + S);
    const uint32_t k = e[0];
    if (k == kEmptyKey || k == rid) {
      e[0] = rid;
#pragma unroll
      for (int s = 0; s < S; ++s) e[1 + s] = w[s];
      if (i) hdr->collisions += i;
      probes = i + 1;
      break;
    }
  }
  if (!probes) hdr->error = 1u;
  __threadfence();
  atomicExch(&hdr->lock, 0u);
  return probes;
}

// Lookup used by validation (L270: lookups are off the critical path).
// Returns true and the stored record words if rid is present.
template <int S>
__device__ __forceinline__ bool quad_lookup(const uint32_t* ckbuf, uint32_t rid, uint32_t* w) {
  const HashHeader* hdr = reinterpret_cast<const HashHeader*>(ckbuf);
  const uint32_t* ent = ckbuf + sizeof(HashHeader) / 4;
  const uint32_t cap = hdr->cap;
  const uint32_t home = hash_fmix32(rid, hdr->seed) % cap;
  for (uint32_t i = 0; i < cap; ++i) {
    const uint32_t slot = (uint32_t)(((uint64_t)home + (uint64_t)i * i) % cap);
    const uint32_t* e = ent + (uint64_t)slot * (1 + S);
    const uint32_t k = e[0];
    if (k == rid) {
#pragma unroll
      for (int s = 0; s < S; ++s) w[s] = e[1 + s];
      return true;
    }
    if (k == kEmptyKey) return false;
  }
  return false;
}

// ---------------------------------------------------------------------------
// Cuckoo store (L269-274, Fig. 4): two tables T1/T2 with hash functions H1/H2;
// an insert puts the key at T1[H1(k)] and carries whatever it evicts to the other
// table (T2[H2(.)], then T1[H1(.)], ...).  L274: "we use atomic exchange
// (atomicExch()) ... we will always insert the entry to a hash table entry no
// matter whether it is occupied or empty".  An entry is 16 bytes {key, rec0,
// rec1, rec2} exchanged with ONE 128-bit atom.exch so a record always travels with
// its key.  Per-table capacity = smallest prime >= 1.15 R: total load <= 43.5%,
// below the 50% threshold of two-table cuckoo hashing (L270 bounds the load).
// L270: "When a cycle is detected, the cuckoo hash table performs hash tables
// rehashing" (Reading R24): an entry still homeless after max_evict placements is
// parked in a small stash behind T2, and the rehash kernel that follows every
// protected / recovery run (cuckoo_rehash_kernel) rebuilds T1/T2 in place with a
// new seed and re-inserts the stash.  Only a stash overflow loses an entry (error
// flag).  Layout: HashHeader, T1[cap], T2[cap], stash[kCuckooStash].
constexpr int kCuckooMaxEvict = 128;
constexpr int kCuckooStash = 256;

__host__ __device__ __forceinline__ uint32_t cuckoo_h(int t, uint32_t key, uint32_t seed, uint32_t cap) {
  return (t == 0 ? hash_fmix32(key, seed) : hash_fmix32(key, seed * 0x9E3779B9u + 0x7F4A7C15u)) % cap;
}

__device__ __forceinline__ uint4 atom_exch_128(uint4* p, uint4 v) {
  const uint64_t lo = ((uint64_t)v.y << 32) | v.x, hi = ((uint64_t)v.w << 32) | v.z;
  uint64_t olo, ohi;
  asm volatile(
      "{\n\t.reg .b128 d, b;\n\tmov.b128 b, {%2, %3};\n\tatom.global.exch.b128 d, [%4], b;\n\tmov.b128 {%0, %1}, d;\n\t}"
      : "=l"(olo), "=l"(ohi)
      : "l"(lo), "l"(hi), "l"(p)
      : "memory");
  return make_uint4((uint32_t)olo, (uint32_t)(olo >> 32), (uint32_t)ohi, (uint32_t)(ohi >> 32));
}

template <uint32_t MASK>
__device__ __forceinline__ uint4 cuckoo_entry(uint32_t rid, const uint32_t* w) {
  constexpr int S = selem_of(MASK);
  return make_uint4(rid, S > 0 ? w[0] : 0u, S > 1 ? w[1] : 0u, S > 2 ? w[2] : 0u);
}

// Placement walk of one entry (Fig. 4): exchange into T1[H1], carry the occupant to the
// other table, ... .  Returns the number of placements, or 0 when the walk hit the
// eviction bound and the homeless entry went to the stash (rehash pending).
__device__ __forceinline__ uint32_t cuckoo_place(HashHeader* hdr, uint4* tab, uint32_t cap, uint32_t seed, uint4 e,
                                                 int bound, bool count) {
  int t = 0;
  for (int i = 0; i < bound; ++i) {
    const uint4 old = atom_exch_128(tab + (uint64_t)t * cap + cuckoo_h(t, e.x, seed, cap), e);
    if (old.x == kEmptyKey || old.x == e.x) {  // empty slot, or the same key's stale entry (dropped)
      if (i && count) atomicAdd(&hdr->collisions, (unsigned long long)i);
      return (uint32_t)i + 1;
    }
    e = old;  // carry the evicted entry to its slot in the other table
    t ^= 1;
  }
  const uint32_t k = atomicAdd(&hdr->stash_n, 1u);
  if (k < (uint32_t)kCuckooStash) {
    uint4* stash = tab + 2ull * cap;
    stash[k] = e;
  } else {
    atomicExch(&hdr->error, 1u);  // stash full: this entry is lost
  }
  return 0;
}

template <uint32_t MASK>
__device__ __forceinline__ uint32_t cuckoo_insert(uint32_t* ckbuf, uint32_t rid, const uint32_t* w) {
  HashHeader* hdr = reinterpret_cast<HashHeader*>(ckbuf);
  uint4* tab = reinterpret_cast<uint4*>(ckbuf + sizeof(HashHeader) / 4);
  const uint32_t cap = hdr->cap, seed = hdr->seed;
  uint4 e = cuckoo_entry<MASK>(rid, w);
  // Re-insertion (recovery): if the key already lives in one of its two slots, replace that
  // entry in place -- inserting at T1 again could leave a stale duplicate in T2 that a later
  // eviction chain would write back over the fresh record.
  for (int t = 0; t < 2; ++t) {
    uint4* slot = tab + (uint64_t)t * cap + cuckoo_h(t, rid, seed, cap);
    if (slot->x == rid) {
      const uint4 old = atom_exch_128(slot, e);
      if (old.x == rid) return 1;
      e = old;  // raced with a concurrent move: carry what we displaced
      if (e.x == kEmptyKey) return 1;
      break;
    }
  }
  const uint32_t me = hdr->max_evict;
  return cuckoo_place(hdr, tab, cap, seed, e, me ? (int)me : kCuckooMaxEvict, true);
}

template <uint32_t MASK>
__device__ __forceinline__ uint32_t cuckoo_insert_locked(uint32_t* ckbuf, uint32_t rid, const uint32_t* w) {
  HashHeader* hdr = reinterpret_cast<HashHeader*>(ckbuf);
  while (atomicCAS(&hdr->lock, 0u, 1u) != 0u) __nanosleep(32);
  __threadfence();
  const uint32_t r = cuckoo_insert<MASK>(ckbuf, rid, w);
  __threadfence();
  atomicExch(&hdr->lock, 0u);
  return r;
}

template <int S>
__device__ __forceinline__ bool cuckoo_lookup(const uint32_t* ckbuf, uint32_t rid, uint32_t* w) {
  const HashHeader* hdr = reinterpret_cast<const HashHeader*>(ckbuf);
  const uint4* tab = reinterpret_cast<const uint4*>(ckbuf + sizeof(HashHeader) / 4);
  const uint32_t cap = hdr->cap, seed = hdr->seed;
  for (int t = 0; t < 2; ++t) {
    const uint4 e = tab[(uint64_t)t * cap + cuckoo_h(t, rid, seed, cap)];
    if (e.x == rid) {
      if (S > 0) w[0] = e.y;
      if (S > 1) w[1] = e.z;
      if (S > 2) w[2] = e.w;
      return true;
    }
  }
  return false;
}

// Record store, selected at compile time so the array-store kernels carry no
// hash-table code (and no register pressure from it).
// STORE: 0 array, 1 quad CAS, 2 quad + global lock, 3 cuckoo (atomicExch), 4 cuckoo + global lock.
template <uint32_t MASK, int STORE>
__device__ __forceinline__ void store_record(uint32_t* ck, int64_t local_rid, uint32_t global_rid, const uint32_t* w) {
  if constexpr (STORE == 0) {
    store_array<MASK>(ck, local_rid, w);
  } else if constexpr (STORE == 1) {
    quad_insert<MASK>(ck, global_rid, w);
  } else if constexpr (STORE == 2) {
    quad_insert_locked<MASK>(ck, global_rid, w);
  } else if constexpr (STORE == 3) {
    cuckoo_insert<MASK>(ck, global_rid, w);
  } else {
    cuckoo_insert_locked<MASK>(ck, global_rid, w);
  }
}

// Lookup dispatch for validation: returns false if the key is absent.
template <int S, int STORE>
__device__ __forceinline__ bool store_lookup(const uint32_t* ck, uint32_t global_rid, uint32_t* w) {
  if constexpr (STORE == 3 || STORE == 4) {
    return cuckoo_lookup<S>(ck, global_rid, w);
  } else {
    return quad_lookup<S>(ck, global_rid, w);
  }
}

// ---------------------------------------------------------------------------
// NVLS-fused failed count: the CTA that finalises a shard's failed
// count also adds it, with multimem.red, into a counter bound to a multicast object that every
// rank maps (NVSwitch performs the reduction into each GPU's copy), bumps an arrival counter the
// same way, and waits until all world_size ranks of this epoch have arrived: every rank then
// holds the all-rank count without a separate NCCL all-reduce launch.  Counter buffer (u64,
// zero-filled once on every rank, symmetric): [0],[1] cumulative counts by epoch parity,
// [2] arrivals, [3] this rank's epoch, [4] RESULT (the all-rank count of the latest epoch),
// [5],[6] last cumulative value by parity.  mc == uc with world == 1 is the single-GPU
// emulation (plain atomics on the local copy) that tests the epoch logic without NVLink.
struct NvlsCount {
  unsigned long long* mc;  // multicast address of the counter buffer (null: feature off)
  unsigned long long* uc;  // this rank's unicast address of the same buffer
  int world;
};

__device__ __forceinline__ void nvls_publish(const NvlsCount& nv, int64_t n) {
  if (nv.uc == nullptr) return;
  volatile unsigned long long* uc = nv.uc;
  const unsigned long long e = uc[3] + 1ull;
  uc[3] = e;
  const int par = (int)(e & 1ull);
  if (nv.mc == nv.uc) {
    atomicAdd(nv.uc + par, (unsigned long long)n);
    __threadfence();
    atomicAdd(nv.uc + 2, 1ull);
  } else {
    asm volatile("multimem.red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(nv.mc + par), "l"((unsigned long long)n)
                 : "memory");
    asm volatile("multimem.red.release.sys.global.add.u64 [%0], %1;" ::"l"(nv.mc + 2), "l"(1ull) : "memory");
  }
  const unsigned long long target = e * (unsigned long long)nv.world;
  unsigned long long arrived;
  for (;;) {
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(arrived) : "l"(nv.uc + 2) : "memory");
    if (arrived >= target) break;
    __nanosleep(64);
  }
  unsigned long long cum;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(cum) : "l"(nv.uc + par) : "memory");
  uc[4] = cum - uc[5 + par];
  uc[5 + par] = cum;
}

// Streaming 16-byte load that does not allocate in L1 (validate reads `out` once).
__device__ __forceinline__ uint4 ld_stream_u4(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

}  // namespace lp
