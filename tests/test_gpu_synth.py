"""The device input generator (lpsynth/synth.cu) reproduces lpsynth/gen.py bit-exactly."""
import numpy as np
import pytest
import torch

import lpsynth
from lpsynth import gen
from tests.gpu_util import dev_to_host

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("kind", ["uniform", "int5", "int17", "bits"])
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_device_fill_matches_host(kind, dtype):
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    t = torch.empty((96, 200), dtype=tdt, device="cuda")
    lpsynth.device_fill(t, 5, kind, dtype, row0=64, ncols_global=200)
    torch.cuda.synchronize()
    ref = gen.generate(5, 96, 200, kind, dtype, row0=64, ncols_global=200)
    assert np.array_equal(dev_to_host(t).view(np.uint8), np.ascontiguousarray(ref).view(np.uint8))
