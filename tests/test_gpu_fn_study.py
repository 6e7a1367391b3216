"""N3 false-negative study kernel: per-trial detection bits re-checked by the CPU oracle on fully
materialised regions, plus the closed-form facts of each corruption model."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
from lpsynth import gen
from paper_conf_iiswc_yudhakzs20_b200 import lp

pytestmark = pytest.mark.gpu

NW = 1024  # a 32x32 fp32 region


def _run(model, kmax, trials, dump_trials, seed=11):
    h = lp.LP(32, 32, cksum="mod|xor|adler")
    counts = torch.zeros(7, dtype=torch.int64, device="cuda")
    dump = torch.zeros(max(dump_trials, 1) * 26, dtype=torch.int32, device="cuda")
    h.fn_study(model, kmax, NW, seed, trials, counts, dump if dump_trials else None, dump_trials)
    torch.cuda.synchronize()
    return counts.cpu().numpy(), dump.cpu().numpy().view(np.uint32).reshape(-1, 26)[:dump_trials]


@pytest.mark.parametrize("model,kmax", [("random_words", 4), ("bitflips", 3), ("adversarial", 2), ("zeroed", 8)])
def test_dumped_trials_match_oracle(model, kmax):
    counts, dump = _run(model, kmax, 20000, 1500)
    assert counts[0] + counts[6] == 20000
    base = gen.generate(99, 32, 32, "bits", "u32")        # region content outside the corrupted words
    for t in range(len(dump)):
        k = int(dump[t, 0])
        pos, old, new = dump[t, 1:1 + k], dump[t, 9:9 + k], dump[t, 17:17 + k]
        before = base.copy().reshape(-1)
        before[pos] = old
        after = before.copy()
        after[pos] = new
        r0 = oracle.records(before.reshape(32, 32), 32, 32, 7)[0]
        r1 = oracle.records(after.reshape(32, 32), 32, 32, 7)[0]
        exp = (int(r0[0] != r1[0]) | (int(r0[1] != r1[1]) << 1) | (int(r0[2] != r1[2]) << 2) |
               (8 if not np.array_equal(before, after) else 0))
        assert int(dump[t, 25]) == exp, (t, int(dump[t, 25]), exp)


def test_model_closed_forms():
    c, _ = _run("adversarial", 2, 100000, 0)
    assert c[6] == 0 and c[1] == c[0] and c[2] == c[0] and c[3] == c[0]   # MOD and XOR blind by construction
    assert c[4] < c[0] // 1000                                           # Adler is position-weighted
    c, _ = _run("bitflips", 1, 100000, 0)
    assert c[1] == 0 and c[2] == 0 and c[4] == 0                          # a single flip changes every checksum
    c, _ = _run("random_words", 1, 100000, 0)
    assert c[3] == 0                                                       # one changed word never hits MOD and XOR
