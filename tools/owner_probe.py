"""Which chain bounds a dilated nest?  Device time of B=256 T=100 H=512 nests that share C4's
layer 0 but differ above it, with the layer-0 owner variants (development aid):
  [1, T]              layer 0's chain + one depth consumer (no recurrence above layer 0)
  [1, T, T, T, T, T]  C4's tile count, no recurrence above layer 0
  C4 [1, 2, 4, 8, 16, 32]
variants: split owners (default), FT_OWNER_SPLIT=0, FT_OWNER_L0=0 (round-robin)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import ftgen  # noqa: E402
from paper_conf_sosp_liuqc0hs0y24_b200 import ft  # noqa: E402

B, T, H = 256, 100, 512
REPS = int(os.environ.get("QT_REPS", "20"))
nests = {"[1,T]": [1, T], "[1,T x5]": [1, T, T, T, T, T], "C4": [1, 2, 4, 8, 16, 32]}
if os.environ.get("PROBE_NESTS"):
    nests = {k: v for k, v in nests.items() if k in os.environ["PROBE_NESTS"].split(";")}
variants = {"split": {}, "plain": {"FT_OWNER_SPLIT": "0"}, "rr": {"FT_OWNER_L0": "0"}}
ws = ft.Workspace()
for name, dil in nests.items():
    p = ftgen.stacked_inputs(B, T, H, len(dil), 1, "bf16")
    a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
    for _ in range(2):
        for vn, env in variants.items():
            for k in ("FT_OWNER_SPLIT", "FT_OWNER_L0"):
                os.environ.pop(k, None)
            os.environ.update(env)
            fn = lambda: ft.stacked_lstm(*a, dilations=dil, workspace=ws)
            for _ in range(3):
                fn()
            torch.cuda.synchronize()
            ts = []
            for _ in range(REPS):
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record(); fn(); e.record(); torch.cuda.synchronize()
                ts.append(s.elapsed_time(e))
            last = ft.ft_last_launch()
            tag = "split" if "split_owner=1" in last else ("owner" if "owner=2" in last else "rr")
            print(f"{name:10s} {vn:6s} ({tag:5s}) median {np.median(ts) * 1e3:7.1f} us  min {np.min(ts) * 1e3:7.1f} us"
                  f"  per step {np.median(ts) * 1e3 / T:5.2f} us", flush=True)
