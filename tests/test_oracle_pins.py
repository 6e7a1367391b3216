"""Pins of the CPU oracle against things other than itself (CPU only).

Each pin is chosen so that a plausible mistake in oracle/lp_oracle.c (a dropped
term, a wrong index/offset, a swapped byte order, a wrong sign or coefficient)
fails at least one test:
  * paper worked examples (tests/golden/*, each with its PAPER.md citation),
  * library routines (zlib.adler32, numpy float64 matmul, torch bf16 rounding),
  * brute force with Python integers on tiny regions,
  * closed forms and invariants.
"""
from __future__ import annotations

import os
import random
import struct
import zlib

import numpy as np
import pytest

import oracle
from lpsynth import gen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


# --------------------------------------------------------------------------- Fig. 2 / Reading R2
def test_fig2_ordered_integer_worked_example():
    (val, expect), = _golden("fig2_float_word.txt")
    assert oracle.float_word(float(val)) == int(expect)
    # The order-preserving sign-flip map would give 3227516928 instead (rejected reading).
    assert oracle.float_word(3.5) != 3227516928


def test_float_word_matches_struct():
    rng = np.random.default_rng(0)
    for v in rng.standard_normal(64).astype(np.float32):
        assert oracle.float_word(float(v)) == struct.unpack("<I", struct.pack("<f", float(v)))[0]


# --------------------------------------------------------------------------- Adler-32 (L192)
def test_adler32_textbook_vector():
    (text, hexv), = _golden("adler32_vectors.txt")
    assert oracle.adler32(text.encode()) == int(hexv, 16)


@pytest.mark.parametrize("n", [0, 1, 2, 255, 5552, 5553, 65536, 100_003])
def test_adler32_vs_zlib(n):
    data = np.random.default_rng(n).integers(0, 256, n, dtype=np.uint8).tobytes()
    assert oracle.adler32(data) == zlib.adler32(data)


def test_adler32_zero_closed_form():
    for n in [1, 7, 65521, 70000]:
        assert oracle.adler32(bytes(n)) == (((n % 65521) << 16) | 1)


# --------------------------------------------------------------------------- region records, brute force
def _words_fp32(block):
    return [struct.unpack("<I", struct.pack("<f", float(v)))[0] for v in block.reshape(-1)]


def _words_bf16(block):
    b = block.reshape(block.shape[0], -1)
    out = []
    for i in range(b.shape[0]):
        for j in range(0, b.shape[1], 2):
            out.append(int(b[i, j]) | (int(b[i, j + 1]) << 16))
    return out


def _brute_record(block, mask):
    words = _words_fp32(block) if block.dtype == np.float32 else _words_bf16(block)
    mod = sum(words) % (1 << 32)
    x = 0
    for w in words:
        x ^= w
    rec = []
    if mask & 1:
        rec.append(mod)
    if mask & 2:
        rec.append(x)
    if mask & 4:
        rec.append(zlib.adler32(np.ascontiguousarray(block).tobytes()))
    return rec


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("RM,RN", [(1, 2), (2, 2), (4, 4), (4, 8), (3, 6)])
def test_records_brute_force(dtype, RM, RN):
    M, N = RM * 3, RN * 2
    out = gen.generate(7, M, N, "uniform", dtype)
    for mask in [1, 2, 4, 3, 7]:
        recs = oracle.records(out, RM, RN, mask)
        Q = N // RN
        for p in range(M // RM):
            for q in range(Q):
                blk = out[p * RM:(p + 1) * RM, q * RN:(q + 1) * RN]
                assert list(recs[p * Q + q]) == _brute_record(np.ascontiguousarray(blk), mask), (p, q, mask)


def test_record_order_and_width():
    out = gen.generate(3, 4, 4, "uniform", "f32")
    r7 = oracle.records(out, 4, 4, 7)[0]
    assert list(oracle.records(out, 4, 4, 1)[0]) == [r7[0]]
    assert list(oracle.records(out, 4, 4, 2)[0]) == [r7[1]]
    assert list(oracle.records(out, 4, 4, 4)[0]) == [r7[2]]
    assert list(oracle.records(out, 4, 4, 5)[0]) == [r7[0], r7[2]]


def test_bf16_word_is_memory_image_even_column_low():
    out = np.array([[0x1111, 0x2222]], dtype=np.uint16)
    (mod, xr), = oracle.records(out, 1, 2, 3)
    assert mod == 0x22221111 and xr == 0x22221111


def test_records_closed_forms():
    # n equal words v: MOD = n*v mod 2^32, XOR = v (n odd) or 0 (n even); zeros -> 0, 0, (nbytes<<16)|1
    v = np.float32(-1.75)
    w = oracle.float_word(float(v))
    for RM, RN in [(3, 3), (4, 4), (32, 32)]:
        out = np.full((RM, RN), v, dtype=np.float32)
        n = RM * RN
        mod, xr, ad = oracle.records(out, RM, RN, 7)[0]
        assert mod == (n * w) % (1 << 32)
        assert xr == (w if n % 2 else 0)
        z = np.zeros((RM, RN), dtype=np.float32)
        assert list(oracle.records(z, RM, RN, 7)[0]) == [0, 0, ((4 * n % 65521) << 16) | 1]


def test_mod_xor_permutation_invariant_adler_not():
    out = gen.generate(11, 8, 8, "uniform", "f32")
    perm = out.reshape(-1).copy()
    np.random.default_rng(1).shuffle(perm)
    perm = perm.reshape(8, 8)
    a = oracle.records(out, 8, 8, 7)[0]
    b = oracle.records(perm, 8, 8, 7)[0]
    assert a[0] == b[0] and a[1] == b[1]
    assert a[2] != b[2]


def test_region_indexing_uses_pitch_and_offsets():
    # record of region (p,q) inside the full matrix == record of the extracted block as a 1-region matrix
    out = gen.generate(5, 96, 160, "uniform", "bf16")
    recs = oracle.records(out, 32, 32, 7)
    Q = 160 // 32
    for p in range(3):
        for q in range(5):
            blk = np.ascontiguousarray(out[p * 32:(p + 1) * 32, q * 32:(q + 1) * 32])
            assert list(recs[p * Q + q]) == list(oracle.records(blk, 32, 32, 7)[0])


def test_single_change_moves_only_its_record():
    out = gen.generate(9, 64, 64, "uniform", "f32")
    base = oracle.records(out, 16, 16, 3)
    bad = out.copy()
    bad[37, 22] = np.float32(bad[37, 22] + 1.0)
    after = oracle.records(bad, 16, 16, 3)
    diff = np.nonzero((base != after).any(axis=1))[0]
    assert list(diff) == [(37 // 16) * 4 + 22 // 16]


# --------------------------------------------------------------------------- validation (L183)
def test_validate_clean_and_corrupted():
    out = gen.generate(2, 128, 128, "uniform", "f32")
    mask = 3
    table = oracle.records(out, 32, 32, mask)
    assert oracle.validate_array(out, table, 32, 32, mask).size == 0
    bad = out.copy()
    w = bad.view(np.uint32)
    w[70, 100] ^= np.uint32(1 << 13)                      # bit flip in region (2,3) = rid 11
    t2 = table.copy()
    t2[5] = oracle.SENTINEL                               # stale record, data intact: rid 5
    got = oracle.validate_array(bad, t2, 32, 32, mask, rid_offset=1000)
    assert list(got) == [1005, 1011]


def test_validate_sentinel_table_fails_everything():
    out = gen.generate(4, 64, 64, "uniform", "bf16")
    table = np.full((16, 2), oracle.SENTINEL, dtype=np.uint32)
    assert list(oracle.validate_array(out, table, 16, 16, 3)) == list(range(16))


# --------------------------------------------------------------------------- TMM body (Listings 2/6)
def test_gemm_identity_and_ones():
    K = 48
    B = gen.generate(1, K, 40, "uniform", "f32")
    I = np.eye(K, dtype=np.float32)
    C = oracle.gemm_block_f64(I, B, 0, 0, K, 40)
    assert np.array_equal(C, B.astype(np.float64))
    ones_a = np.ones((16, K), dtype=np.float32)
    ones_b = np.ones((K, 24), dtype=np.float32)
    assert np.all(oracle.gemm_block_f64(ones_a, ones_b, 0, 0, 16, 24) == K)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_gemm_vs_numpy_float64(dtype):
    A = gen.generate(1, 64, 96, "uniform", dtype)
    B = gen.generate(2, 96, 80, "uniform", dtype)
    to64 = (lambda x: x.astype(np.float64)) if dtype == "f32" else (lambda x: oracle.bf16_bits_to_f32(x).astype(np.float64))
    ref = to64(A) @ to64(B)
    got = oracle.gemm_block_f64(A, B, 16, 32, 32, 48)
    assert np.allclose(got, ref[16:48, 32:80], rtol=1e-12, atol=1e-12)


def test_gemm_integer_valued_exact():
    A = gen.generate(3, 32, 256, "int5", "f32")
    B = gen.generate(4, 256, 32, "int5", "f32")
    ref = A.astype(np.int64) @ B.astype(np.int64)
    got = oracle.gemm_block_f64(A, B, 0, 0, 32, 32)
    assert np.array_equal(got.astype(np.int64), ref)


def test_round_bf16_vs_torch():
    torch = pytest.importorskip("torch")
    rng = np.random.default_rng(0)
    x = np.concatenate([rng.standard_normal(5000) * 1000, np.arange(-40000, 40000, 7, dtype=np.float64)])
    # exact ties: values halfway between two bf16 numbers
    ties = (np.arange(1, 200, dtype=np.float64) * 2 + 1) * 2.0 ** 9  # odd multiples of 2^9 in [2^16..] -> ties
    x = np.concatenate([x, ties])
    got = oracle.round_bf16(x)
    ref = torch.from_numpy(x.astype(np.float32)).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(got, ref)


# --------------------------------------------------------------------------- stencil body (Reading R19)
def test_stencil_impulse_response():
    x = np.zeros((7, 9), dtype=np.float32)
    x[3, 4] = 1.0
    y = oracle.stencil5(x)
    expect = np.zeros_like(x)
    expect[3, 4] = 0.5
    for di, dj in [(-1, 0), (1, 0), (0, -1), (0, 1)]:
        expect[3 + di, 4 + dj] = 0.125
    assert np.array_equal(y, expect)


def test_stencil_constant_closed_form():
    c = np.float32(3.0)
    y = oracle.stencil5(np.full((6, 5), c, dtype=np.float32))
    assert np.all(y[1:-1, 1:-1] == c)
    assert y[0, 0] == np.float32(0.75) * c and y[-1, -1] == np.float32(0.75) * c
    assert np.all(y[0, 1:-1] == np.float32(0.875) * c) and np.all(y[1:-1, 0] == np.float32(0.875) * c)


def test_stencil_quadratic_closed_form():
    # in = i^2 + 3 j^2  =>  interior out = in + 0.125*(2 + 6) = in + 1 (exact for these integers)
    i = np.arange(20, dtype=np.float32)[:, None]
    j = np.arange(17, dtype=np.float32)[None, :]
    x = (i * i + 3 * j * j).astype(np.float32)
    y = oracle.stencil5(x)
    assert np.array_equal(y[1:-1, 1:-1], x[1:-1, 1:-1] + 1)


def test_stencil_block_matches_full():
    x = gen.generate(8, 40, 36, "uniform", "f32")
    full = oracle.stencil5(x)
    assert np.array_equal(oracle.stencil5_block(x, 8, 12, 16, 12), full[8:24, 12:24])


# --------------------------------------------------------------------------- quadratic probing (L267)
def test_quad_probe_offsets_match_paper_example():
    cap = 101
    rows = _golden("quad_probe_example.txt")
    for key in [0, 5, 77, 12345]:
        h = oracle.quad_hash(key, 0, cap)
        for i, off in rows:
            assert oracle.quad_probe(key, 0, cap, int(i)) == (h + int(off)) % cap


def test_quad_hash_is_murmur_fmix32():
    def fmix(h):
        h ^= h >> 16
        h = (h * 0x85EBCA6B) & 0xFFFFFFFF
        h ^= h >> 13
        h = (h * 0xC2B2AE35) & 0xFFFFFFFF
        h ^= h >> 16
        return h
    for key in [0, 1, 2, 1000, 2 ** 31 + 5]:
        assert oracle.quad_hash(key, 0x9747B28C, 4099) == fmix(key ^ 0x9747B28C) % 4099


def test_quad_insert_lookup_roundtrip_at_load_07():
    R, sel, seed = 700, 2, 17
    cap = 1009  # prime >= R/0.7
    table = np.full(cap * (1 + sel), 0xFFFFFFFF, dtype=np.uint32)
    rng = random.Random(0)
    recs = {k: [rng.getrandbits(32), rng.getrandbits(32)] for k in range(R)}
    total_probes = 0
    for k in range(R):
        n = oracle.quad_insert(table, cap, sel, k, seed, recs[k])
        assert n >= 1
        total_probes += n
    keys = table.reshape(cap, 1 + sel)[:, 0]
    assert np.sum(keys != 0xFFFFFFFF) == R and len(set(keys[keys != 0xFFFFFFFF].tolist())) == R
    for k in range(R):
        assert list(oracle.quad_lookup(table, cap, sel, k, seed)) == recs[k]
    assert oracle.quad_lookup(table, cap, sel, R + 5, seed) is None
    assert total_probes > R  # at load 0.7 collisions happen (Table II)


def test_validate_quad_missing_key_is_failed():
    out = gen.generate(6, 64, 64, "uniform", "f32")
    RM = RN = 32
    recs = oracle.records(out, RM, RN, 3)
    cap, seed = 7, 3
    table = np.full(cap * 3, 0xFFFFFFFF, dtype=np.uint32)
    for rid in [0, 1, 3]:                 # rid 2 never inserted
        oracle.quad_insert(table, cap, 2, rid, seed, recs[rid])
    assert list(oracle.validate_quad(out, table, cap, seed, RM, RN, 3)) == [2]


# --------------------------------------------------------------------------- synthetic inputs
def test_splitmix64_reference_vector():
    # splitmix64 with state 0: first output 0xE220A8397B1DCDAF (Vigna's reference implementation)
    assert int(gen.splitmix64(np.array([0], dtype=np.uint64))[0]) == 0xE220A8397B1DCDAF


def test_synth_value_ranges_and_shard_invariance():
    u = gen.generate(1, 64, 64, "uniform", "f32")
    assert u.min() >= -1 and u.max() < 1 and np.all((u.astype(np.float64) * 2 ** 23) % 1 == 0)
    i5 = gen.generate(1, 64, 64, "int5", "f32")
    assert set(np.unique(i5).tolist()) <= {-2, -1, 0, 1, 2}
    full = gen.generate(3, 32, 48, "uniform", "bf16")
    shard = gen.generate(3, 8, 48, "uniform", "bf16", row0=16, ncols_global=48)
    assert np.array_equal(full[16:24], shard)


def test_synth_column_block_matches_full():
    full = gen.generate(4, 16, 40, "int5", "bf16")
    blk = gen.generate(4, 16, 8, "int5", "bf16", ncols_global=40, col0=24)
    assert np.array_equal(full[:, 24:32], blk)


def test_gemm_int32_operands_vs_numpy_int64():
    A = gen.generate(3, 32, 128, "int17", "i32")
    B = gen.generate(4, 128, 48, "int5", "i32")
    assert A.dtype == np.int32
    ref = A.astype(np.int64) @ B.astype(np.int64)
    got = oracle.gemm_block_f64(A, B, 0, 16, 32, 32)
    assert np.array_equal(got.astype(np.int64), ref[:, 16:48])



# --------------------------------------------------------------------------- cuckoo hashing (L269-270)
def test_cuckoo_hashes_re_derived():
    def fmix(h):
        h ^= h >> 16
        h = (h * 0x85EBCA6B) & 0xFFFFFFFF
        h ^= h >> 13
        h = (h * 0xC2B2AE35) & 0xFFFFFFFF
        h ^= h >> 16
        return h
    seed, cap = 0x9747B28C, 1009
    for key in [0, 7, 123456]:
        assert oracle.cuckoo_hash(0, key, seed, cap) == fmix(key ^ seed) % cap
        assert oracle.cuckoo_hash(1, key, seed, cap) == fmix(key ^ ((seed * 0x9E3779B9 + 0x7F4A7C15) & 0xFFFFFFFF)) % cap


def test_cuckoo_eviction_moves_occupant_to_other_table():
    # Fig. 4 step (1)-(2): X hashes onto C's T1 slot -> X takes it, C moves to T2[H2(C)]
    cap, seed = 101, 5
    tab = np.full(2 * cap * 4, 0xFFFFFFFF, dtype=np.uint32)
    c = 3
    x = next(k for k in range(4, 100000) if oracle.cuckoo_hash(0, k, seed, cap) == oracle.cuckoo_hash(0, c, seed, cap))
    assert oracle.cuckoo_insert(tab, cap, 1, c, seed, [111]) == 1
    assert oracle.cuckoo_insert(tab, cap, 1, x, seed, [222]) == 2
    t1 = tab.reshape(2, cap, 4)
    assert t1[0, oracle.cuckoo_hash(0, x, seed, cap), 0] == x
    assert t1[1, oracle.cuckoo_hash(1, c, seed, cap), 0] == c
    assert list(oracle.cuckoo_lookup(tab, cap, 1, c, seed)) == [111]
    assert list(oracle.cuckoo_lookup(tab, cap, 1, x, seed)) == [222]


def _nextprime(c):
    while c < 2 or any(c % d == 0 for d in range(2, int(c ** 0.5) + 1)):
        c += 1
    return c


def test_cuckoo_roundtrip_at_library_sizing():
    R, sel, seed = 1000, 2, 9
    cap = _nextprime(int(np.ceil(R * 1.15)))  # liblp's per-table sizing: total load 1000 / 2302 = 43% (L270)
    tab = np.full(2 * cap * 4, 0xFFFFFFFF, dtype=np.uint32)
    rng = random.Random(1)
    recs = {k: [rng.getrandbits(32), rng.getrandbits(32)] for k in range(R)}
    evictions = 0
    for k in range(R):
        n = oracle.cuckoo_insert(tab, cap, sel, k, seed, recs[k])
        assert n >= 1
        evictions += n - 1
    keys = tab.reshape(2 * cap, 4)[:, 0]
    present = keys[keys != 0xFFFFFFFF]
    assert len(present) == R and len(set(present.tolist())) == R
    for k in range(R):
        assert list(oracle.cuckoo_lookup(tab, cap, sel, k, seed)) == recs[k]
    assert oracle.cuckoo_lookup(tab, cap, sel, R + 3, seed) is None
    assert evictions > 0



def test_cuckoo_reinsert_updates_in_place():
    cap, seed = 53, 2
    tab = np.full(2 * cap * 4, 0xFFFFFFFF, dtype=np.uint32)
    for k in range(40):
        oracle.cuckoo_insert(tab, cap, 2, k, seed, [k, k + 1])
    for k in range(40):                       # recovery re-inserts every key with a new record
        oracle.cuckoo_insert(tab, cap, 2, k, seed, [7 * k, 9])
    keys = tab.reshape(2 * cap, 4)[:, 0]
    assert np.sum(keys != 0xFFFFFFFF) == 40   # no duplicates
    for k in range(40):
        assert list(oracle.cuckoo_lookup(tab, cap, 2, k, seed)) == [7 * k, 9]


# --------------------------------------------------------------------------- hand-built hash tables (L183)
def _fmix32(h):
    h ^= h >> 16
    h = (h * 0x85EBCA6B) & 0xFFFFFFFF
    h ^= h >> 13
    h = (h * 0xC2B2AE35) & 0xFFFFFFFF
    h ^= h >> 16
    return h


def _records_by_hand(out, RM, RN, mask):
    """{local rid: record} from Python ints + zlib (no oracle call)."""
    Q = out.shape[1] // RN
    return {p * Q + q: _brute_record(np.ascontiguousarray(out[p * RM:(p + 1) * RM, q * RN:(q + 1) * RN]), mask)
            for p in range(out.shape[0] // RM) for q in range(Q)}


def test_validate_cuckoo_hand_built_table():
    """lpo_validate_cuckoo against a T1/T2 table placed by hand (L269-270, Fig. 4; Reading R24), with a global
    rid offset: one key missing, one record word wrong, one key living in T2 and one region whose data changed.
    The expected failed list is written out by hand below."""
    RM = RN = 4
    out = gen.generate(21, 16, 16, "uniform", "f32")          # 4 x 4 regions, local rids 0..15
    mask, sel, seed, cap, off = 3, 2, 0x1234567, 211, 100
    h2seed = (seed * 0x9E3779B9 + 0x7F4A7C15) & 0xFFFFFFFF
    tab = np.full((2, cap, 4), 0xFFFFFFFF, dtype=np.uint32)
    recs = _records_by_hand(out, RM, RN, mask)
    for rid, rec in recs.items():
        if rid == 5:                                          # never persisted (missing key)
            continue
        key = rid + off                                       # hash stores key on the GLOBAL rid
        s1, s2 = _fmix32(key ^ seed) % cap, _fmix32(key ^ h2seed) % cap
        t, s = (1, s2) if (rid == 12 or tab[0, s1, 0] != 0xFFFFFFFF) else (0, s1)   # rid 12 forced into T2
        assert tab[t, s, 0] == 0xFFFFFFFF
        tab[t, s] = [key] + rec + [0]
    def slot_of(key):
        for t, hs in ((0, seed), (1, h2seed)):
            s = _fmix32(key ^ hs) % cap
            if tab[t, s, 0] == key:
                return t, s
        return None
    t9, s9 = slot_of(off + 9)                                 # rid 9: XOR word of its record is wrong
    tab[t9, s9, 2] ^= 0x10
    assert slot_of(off + 12)[0] == 1                          # rid 12 lives in T2
    bad = out.copy()
    bad.view(np.uint32)[13, 9] ^= np.uint32(1 << 30)         # data of region (3, 2) = local rid 14 changed
    got = oracle.validate_cuckoo(bad, tab, cap, seed, RM, RN, mask, rid_offset=off)
    assert list(got) == [105, 109, 114]
    # the clean image with the completed, correct table validates
    tab[t9, s9, 2] ^= 0x10
    s5 = _fmix32(105 ^ seed) % cap
    t5, s5 = (0, s5) if tab[0, s5, 0] == 0xFFFFFFFF else (1, _fmix32(105 ^ h2seed) % cap)
    assert tab[t5, s5, 0] == 0xFFFFFFFF
    tab[t5, s5] = [105] + recs[5] + [0]
    assert list(oracle.validate_cuckoo(out, tab, cap, seed, RM, RN, mask, rid_offset=off)) == []
    # keys placed without the offset (a shard that forgot rid_offset) fail every region
    assert list(oracle.validate_cuckoo(out, tab, cap, seed, RM, RN, mask, rid_offset=0)) == list(range(16))


def test_validate_quad_hand_built_table_with_offset():
    """lpo_validate_quad against a quadratic-probing table placed by hand (home + i^2, L267; Reading R14/R20),
    global rids = local + 1000: a missing key, a wrong MOD word and a key displaced to its 2nd probe slot."""
    RM = RN = 8
    out = gen.generate(22, 32, 16, "uniform", "bf16")   # 4 x 2 regions, local rids 0..7
    mask, sel, seed, cap, off = 3, 2, 77, 13, 1000
    tab = np.full((cap, 1 + sel), 0xFFFFFFFF, dtype=np.uint32)
    recs = _records_by_hand(out, RM, RN, mask)
    for rid, rec in recs.items():
        if rid == 6:                                          # never persisted
            continue
        key = rid + off
        h = _fmix32(key ^ seed) % cap
        for i in range(cap):
            s = (h + i * i) % cap
            if tab[s, 0] == 0xFFFFFFFF:
                tab[s] = [key] + rec
                break
    # rid 2's MOD word is wrong
    h = _fmix32((off + 2) ^ seed) % cap
    s2 = next((h + i * i) % cap for i in range(cap) if tab[(h + i * i) % cap, 0] == off + 2)
    tab[s2, 1] += np.uint32(1)
    got = oracle.validate_quad(out, tab, cap, seed, RM, RN, mask, rid_offset=off)
    assert list(got) == [1002, 1006]
    tab[s2, 1] -= np.uint32(1)
    assert list(oracle.validate_quad(out, tab, cap, seed, RM, RN, mask, rid_offset=off)) == [1006]
    assert list(oracle.validate_quad(out, tab, cap, seed, RM, RN, mask, rid_offset=0)) == list(range(8))


# --------------------------------------------------------------------------- stencil operation order (Reading R19)
def test_stencil_sum_order_crafted():
    """((u + d) + l) + r in fp32, then 0.5*c + 0.125*s: a crafted neighbourhood where the four plausible
    summation orders round differently.  u = 2^24, d = l = 1, r = 2, c = 0 at the centre (1, 1):
      ((u+d)+l)+r: 2^24+1 -> 2^24 (tie, even), +1 -> 2^24, +2 -> 2^24+2;   * 0.125 -> 2097152.25
      (u+d)+(l+r): 2^24+3 -> 2^24+4 (tie, even);                            * 0.125 -> 2097152.5
      ((u+d)+r)+l: 2^24+2, +1 -> 2^24+4 (tie, even);                        * 0.125 -> 2097152.5
      ((l+r)+u)+d: 3+2^24 -> 2^24+4, +1 -> 2^24+4;                          * 0.125 -> 2097152.5"""
    x = np.zeros((3, 3), dtype=np.float32)
    x[0, 1], x[2, 1], x[1, 0], x[1, 2] = 2.0 ** 24, 1.0, 1.0, 2.0
    assert oracle.stencil5(x)[1, 1] == np.float32(2097152.25)
    # centre term added after the scaled sum: c = 1 -> 0.5 + 2097152.25 = 2097152.75 (exact, ulp 0.25)
    x[1, 1] = 1.0
    assert oracle.stencil5(x)[1, 1] == np.float32(2097152.75)
    # u and d are the vertical neighbours: swap roles (l = 2^24 horizontally) -> ((1+1)+2^24)+2 = 2^24+2... and
    # ((u+d)+l)+r with u = d = 1, l = 2^24, r = 2: 2 + 2^24 -> 2^24+2, +2 -> 2^24+4 -> 2097152.5 + 0.5*c
    y = np.zeros((3, 3), dtype=np.float32)
    y[0, 1], y[2, 1], y[1, 0], y[1, 2] = 1.0, 1.0, 2.0 ** 24, 2.0
    assert oracle.stencil5(y)[1, 1] == np.float32(2097152.5)


def test_stencil_random_vs_float32_numpy_in_stated_order():
    """Random fp32 inputs: the oracle equals a numpy float32 evaluation in Reading R19's order (zero outside the
    domain) element for element -- catches a contraction (FMA), a dropped or doubled neighbour, or an index slip."""
    x = gen.generate(23, 37, 29, "uniform", "f32") * np.float32(1000.0)
    p = np.pad(x, 1)
    u, d, l, r, c = p[:-2, 1:-1], p[2:, 1:-1], p[1:-1, :-2], p[1:-1, 2:], p[1:-1, 1:-1]
    s = ((u + d) + l) + r
    ref = np.float32(0.5) * c + np.float32(0.125) * s
    assert ref.dtype == np.float32
    assert np.array_equal(oracle.stencil5(x).view(np.uint32), ref.view(np.uint32))
    alt = np.float32(0.5) * c + np.float32(0.125) * ((u + d) + (l + r))
    assert not np.array_equal(alt.view(np.uint32), ref.view(np.uint32))   # the input does separate the orders
