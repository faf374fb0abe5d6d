"""Print ft_last_launch() for a config (which kernel / schedule the library picks)."""
import sys
import torch
sys.path.insert(0, ".")
import ftgen  # noqa: E402
from paper_conf_sosp_liuqc0hs0y24_b200 import ft  # noqa: E402
for name in sys.argv[1:]:
    c = ftgen.CONFIGS[name]
    if c["kind"] == "grid":
        g = ftgen.grid_inputs(c["batch"], c["len_x"], c["len_y"], c["hidden"], c["depth"], 1, "bf16")
        a = [torch.from_numpy(g[k]).cuda().to(torch.bfloat16) for k in ("x", "ys", "W", "U")] + [torch.from_numpy(g["b"]).cuda()]
        ft.grid_rnn(*a)
    else:
        p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
        a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
        ft.stacked_lstm(*a, dilations=list(c.get("dilations", [])) or None)
    torch.cuda.synchronize()
    print(name, ft.ft_last_launch())
