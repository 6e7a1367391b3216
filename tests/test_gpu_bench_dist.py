"""The N>1 bench path (region-row shards, count all-reduce, max-over-ranks timing) run end to end on a
1-GPU box: 2 ranks over gloo, both on cuda:0 (bench.py --dist-backend gloo --same-device).  Timing is
meaningless here; the test checks that every rank's shard validates and recovers to zero failures and
that rank 0 prints one well-formed line for the whole job."""
from __future__ import annotations

import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_two_rank_bench_same_device():
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29541", "bench.py", "--gpus", "2", "--steps", "2",
           "--warmup", "3", "--overhead-reps", "2", "--no-cpu-baseline", "--dist-backend", "gloo", "--same-device",
           "--workload", "tmm8192_bf16"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["n_failed_after_recover"] == 0
    assert d["config"]["regions_per_rank"] * 2 == (d["config"]["M_global"] // 128) * (d["config"]["N"] // 128)
    assert d["n_failed_per_step"] == 2 * round(0.05 * d["config"]["regions_per_rank"])
    assert d["value"] > 0 and d["roofline"]["achieved"] > 0
    assert d["per_rank"]["n_failed"]["min"] == d["per_rank"]["n_failed"]["max"] == round(0.05 * d["config"]["regions_per_rank"])


def test_self_launch_two_rank_stencil_same_device():
    """`python bench.py --gpus 2` without torchrun re-launches itself with 2 ranks; default
    workload = C4 stencil, weak-scaled by 32768-row bands with read-only halo rows."""
    cmd = [sys.executable, "bench.py", "--gpus", "2", "--steps", "2", "--warmup", "3", "--overhead-reps", "2",
           "--no-cpu-baseline", "--dist-backend", "gloo", "--same-device"]
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["n_failed_after_recover"] == 0 and d["scaling"] == "weak"
    assert d["config"]["workload"] == "stencil32768" and d["config"]["M_global"] == 65536
    assert d["config"]["regions_per_rank"] == 256 * 256
    assert d["n_failed_per_step"] == 2 * round(0.10 * 256 * 256)
    assert d["dtype"].startswith("f32->f32")


def test_inject_skips_rids_of_other_shards():
    """lp_inject takes GLOBAL rids; ids outside this shard's range are skipped (no write, no fault)."""
    import torch

    from paper_conf_iiswc_yudhakzs20_b200 import lp

    M, N, K, reg = 256, 256, 64, 128
    a = torch.ones((M, K), dtype=torch.bfloat16, device="cuda")
    b = torch.ones((K, N), dtype=torch.bfloat16, device="cuda")
    h = lp.LP(reg, reg, cksum="mod|xor")
    wl = lp.Workload.tmm(a, b, out_dtype="bf16", row_offset=512, global_m=1024)   # rids 8..11 of 0..15
    out, ck, failed, d_n, ws = h.alloc(wl)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    stale = torch.zeros_like(out)
    before = out.clone()
    inj = torch.tensor([0, 7, 12, 1 << 40], dtype=torch.int64, device="cuda")   # none in 8..11 (n <= R)
    h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=5)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert torch.equal(out, before) and int(d_n.item()) == 0
    h.inject(wl, out, ck, stale, torch.tensor([9], dtype=torch.int64, device="cuda"), mode="stale_region", seed=5)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 1 and int(failed[0].item()) == 9


def test_two_rank_spmv_bench_same_device():
    """SpMV row-band shards (strong scaling of the 4 Mi-row matrix over 2 ranks, 4-aligned CSR slices)."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29543", "bench.py", "--gpus", "2", "--steps", "2",
           "--warmup", "3", "--overhead-reps", "2", "--no-cpu-baseline", "--dist-backend", "gloo", "--same-device",
           "--workload", "spmv4m"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["n_failed_after_recover"] == 0
    assert d["config"]["regions_per_rank"] == 4194304 // 1024 // 2
    assert d["n_failed_per_step"] == 2 * round(0.10 * 2048)
