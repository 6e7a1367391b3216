"""Small runs of every kernel family for compute-sanitizer (memcheck / racecheck / synccheck)."""
import sys

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402


def cycle(h, wl, out, ck, failed, d_n, ws, stale, frac=0.2):
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    R = h.num_regions(wl)
    inj = torch.from_numpy(lp.choose_regions(R, frac, 5)).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_words", seed=5)
    h.validate(wl, out, ck, failed, d_n, ws)
    h.recover(wl, out, ck, failed, d_n, ws)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0


def tmm(M, N, K, reg, in_dt, out_dt, body, store="array", shuffle=True, **flags):
    tdt = {"bf16": torch.bfloat16, "f32": torch.float32, "i32": torch.int32}[in_dt]
    a = torch.empty((M, K), dtype=tdt, device="cuda")
    b = torch.empty((K, N), dtype=tdt, device="cuda")
    kind = "int5"
    lpsynth.device_fill(a, 1, kind, in_dt)
    lpsynth.device_fill(b, 2, kind, in_dt)
    h = lp.LP(reg, reg, cksum="mod|xor", store=store, body=body, shuffle=shuffle, **flags)
    wl = lp.Workload.tmm(a, b, out_dtype=out_dt)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = torch.zeros_like(out)
    cycle(h, wl, out, ck, failed, d_n, ws, stale)
    print("ok", M, N, K, reg, in_dt, out_dt, body, store, shuffle, flags, flush=True)
    return h, wl, out, ck, stale


def stencil(store="array", cksum="mod|xor", shard=False):
    x = torch.empty((512, 384), dtype=torch.float32, device="cuda")
    lpsynth.device_fill(x, 1, "uniform", "f32")
    h = lp.LP(128, 128, cksum=cksum, store=store)
    # shard: rows 128..383 of the 512-row domain (halo rows above and below read, not written)
    wl = lp.Workload.stencil(x[128:384], row_offset=128, global_m=512) if shard else lp.Workload.stencil(x)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = torch.zeros_like(out)
    cycle(h, wl, out, ck, failed, d_n, ws, stale)
    d_rec = torch.zeros(1, dtype=torch.int64, device="cuda")
    h.check_recover(wl, out, ck, d_rec)
    torch.cuda.synchronize()
    print("ok stencil", store, cksum, shard, flush=True)


def spmv():
    from lpsynth import csr, gen
    rows, RN = 8192, 1024
    rp = csr.row_ptr(5, rows)
    cols = csr.columns(6, rp, rows)
    vals = gen.values_f32(7, 1, int(rp[-1]), "int5")[0]
    x = gen.values_f32(8, 1, rows, "int5")[0]
    h = lp.LP(1, RN, cksum="mod|xor")
    wl = lp.Workload.spmv(torch.from_numpy(vals).cuda(), torch.from_numpy(x).cuda(), torch.from_numpy(rp).cuda(),
                          torch.from_numpy(cols).cuda())
    out, ck, failed, d_n, ws = h.alloc(wl)
    cycle(h, wl, out, ck, failed, d_n, ws, torch.zeros_like(out))
    print("ok spmv", flush=True)


def validate_large_table():
    """R = 65536 > 16384: validate + the separate ordered-compaction launch."""
    out = torch.randn(2048, 4096, device="cuda").to(torch.bfloat16)
    h = lp.LP(32, 32, cksum="mod|xor")
    wl = lp.Workload.tmm(None, None, out_dtype="bf16", m=2048, n=4096, k=16)
    _, ck, failed, d_n, ws = h.alloc(wl)
    h.region_checksums(wl, out, ck)
    ck[1::97] ^= 1
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) > 0
    print("ok validate R =", h.num_regions(wl), flush=True)


tmm(256, 256, 128, 32, "f32", "f32", "simt")
tmm(256, 256, 128, 32, "i32", "i32", "simt", store="cuckoo", shuffle=False)
tmm(256, 512, 128, 128, "bf16", "bf16", "tcgen05")
tmm(256, 512, 128, 32, "bf16", "f32", "tcgen05", store="quad_cas")
tmm(256, 512, 64, 128, "f32", "f32", "tcgen05", store="cuckoo")
stencil()
stencil("quad_cas")
tmm(256, 512, 1024, 128, "f32", "f32", "tcgen05")     # 3xTF32: two 512-K chunks through the TMEM running sum
spmv()
validate_large_table()


# round 2: Listing 7 on the TMM (check phase + DSMEM bitmask merge), cuckoo stash + device rehash,
# 128x128 regions recovered as slices with cross-task record combine, NVLS count (single-GPU emulation)
h, wl, out, ck, stale = tmm(512, 768, 128, 128, "bf16", "bf16", "tcgen05")
inj = torch.from_numpy(lp.choose_regions(h.num_regions(wl), 0.3, 9)).cuda()
h.inject(wl, out, ck, stale, inj, mode="stale_words", seed=9)
d_rec = torch.zeros(1, dtype=torch.int64, device="cuda")
h.check_recover(wl, out, ck, d_rec)
torch.cuda.synchronize()
print("ok tmm check_recover", int(d_rec.item()), flush=True)
tmm(1024, 1024, 64, 32, "bf16", "bf16", "tcgen05", store="cuckoo", cuckoo_short_chains=True)
tmm(512, 1024, 128, 128, "bf16", "bf16", "tcgen05", recover_slices128=True)
h2, wl2, out2, ck2, stale2 = tmm(512, 512, 64, 128, "bf16", "bf16", "tcgen05", nvls_count=True)
cnt = torch.zeros(16, dtype=torch.int64, device="cuda")
h2.attach_nvls_count(cnt, cnt, 1)
_, _, failed2, d_n2, ws2 = h2.alloc(wl2)
h2.validate(wl2, out2, ck2, failed2, d_n2, ws2)
torch.cuda.synchronize()
print("ok nvls emulation", int(cnt[3].item()), flush=True)


# round 2 (late): two-phase stencil epilogue with Adler, TMA-fed stencil recovery on a row shard (halo rows
# through the tensor map's OOB fill), SIMT 32x32 regions on 128x128 CTA tiles with a hash store
stencil(cksum="mod|xor|adler")
stencil(shard=True)
stencil("cuckoo", shard=True)
tmm(256, 384, 64, 32, "i32", "i32", "simt", store="quad_cas")
tmm(256, 384, 64, 32, "bf16", "f32", "simt")
