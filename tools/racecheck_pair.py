"""Small CTA-pair invocations for compute-sanitizer racecheck (development aid)."""
import os, sys
import torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
os.environ["FT_RESIDENT"] = "0"
for B, T, H, D, extra in ((130, 3, 128, 2, {}), (256, 3, 128, 3, {"FT_BAND": "2"}), (130, 3, 128, 2, {"FT_TILE_UNITS": "32"})):
    os.environ.update(extra)
    p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
    a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
    ft.stacked_lstm(*a, want_all=True)
    torch.cuda.synchronize()
    print(ft.ft_last_launch())
    for k in extra:
        os.environ.pop(k)
print("racecheck cases done")
