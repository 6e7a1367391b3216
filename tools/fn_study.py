#!/usr/bin/env python
"""N3: false-negative rates of MOD / XOR / MOD|XOR / ADLER32 under random error injection on the GPU.

usage: python tools/fn_study.py [trials_per_model] > profiles/<round>/fn_study.md
"""
import sys
import time

import torch

sys.path.insert(0, ".")
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

trials = int(float(sys.argv[1])) if len(sys.argv) > 1 else int(4e9)
h = lp.LP(128, 128, cksum="mod|xor|adler")
nw = 128 * 128  # a 128x128 fp32 region
counts = torch.zeros(7, dtype=torch.int64, device="cuda")
print(f"# False-negative study (N3), {trials:.3g} trials per model, region = {nw} words (128x128 fp32)\n")
print("Paper (L192, CPU LP [9]): modular and Adler-32 < 2e-9 each; modular+parity < 1e-12.\n")
print("| model | kmax | changed trials | undetected MOD | XOR | MOD+XOR | ADLER32 | all three | rate MOD | rate MOD+XOR | "
      "rate ADLER | GPU s |")
print("|---|---|---|---|---|---|---|---|---|---|---|---|")
for model, kmax in [("random_words", 1), ("random_words", 8), ("bitflips", 2), ("bitflips", 8), ("zeroed", 8),
                    ("adversarial", 2)]:
    t0 = time.time()
    tot = [0] * 7
    chunk = int(2e9)
    done = 0
    seed = 1
    while done < trials:
        n = min(chunk, trials - done)
        h.fn_study(model, kmax, nw, seed, n, counts)
        torch.cuda.synchronize()
        tot = [a + int(b) for a, b in zip(tot, counts.tolist())]
        done += n
        seed += 1
    dt = time.time() - t0
    eff = max(tot[0], 1)
    print(f"| {model} | {kmax} | {tot[0]:.4g} | {tot[1]} | {tot[2]} | {tot[3]} | {tot[4]} | {tot[5]} | "
          f"{tot[1] / eff:.2e} | {tot[3] / eff:.2e} | {tot[4] / eff:.2e} | {dt:.1f} |", flush=True)
