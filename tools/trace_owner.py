"""Epilogue role cycles per tile of C4's layer-0 owner CTAs vs the other CTAs (trace build)."""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ft.LIB_PATH = os.path.abspath("build/trace/libft_trace.so")
L = ft.lib()
L.ft_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
NAMES = ["P_flag", "P_empty", "M_full", "M_tempty", "E_tfull", "E_work", "E_cflag", "total", "tiles", "E_ldtm", "E_math", "E_store", "E_bar", "E_rel"]
c = ftgen.CONFIGS["C4"]
p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
ws = ft.Workspace()
fn = lambda: ft.stacked_lstm(*a, dilations=list(c["dilations"]), workspace=ws)
for _ in range(3): fn()
buf = (ctypes.c_ulonglong * (1024 * 16))()
L.ft_debug_trace(buf, 1024 * 16, 1)
fn(); torch.cuda.synchronize()
L.ft_debug_trace(buf, 1024 * 16, 1)
arr = np.array(buf[:], dtype=np.float64).reshape(1024, 16)[:148, :14]
print(ft.ft_last_launch())
for label, rows in (("owners (CTAs 0-15)", slice(0, 16, 2)), ("others (leaders)", slice(16, 148, 2))):
    sub = arr[rows]
    tiles = sub[:, 8].mean()
    print(label, "tiles/CTA", tiles, "total cycles", sub[:, 7].mean())
    for i in (0, 1, 2, 3, 4, 5, 9, 10, 11, 12, 13):
        print(f"  {NAMES[i]:9s} {sub[:, i].mean() / max(tiles, 1):9.0f} cycles/tile")
