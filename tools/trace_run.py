"""Role timing of the bf16 wavefront (development aid): loads build/trace/libft_trace.so."""
import ctypes, sys, os, json
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ft.LIB_PATH = os.path.abspath(os.environ.get("FT_TRACE_LIB", "build/trace/libft_trace.so"))
L = ft.lib()
L.ft_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
NAMES = ["P_flag", "P_empty", "M_full", "M_tempty", "E_tfull", "E_work", "E_cflag", "total", "tiles", "E_ldtm", "E_math", "E_store", "E_bar", "E_rel"]
for name in sys.argv[1:] or ["C3"]:
    if ":" in name:  # custom stacked spec  name:B,T,H,D
        B_, T_, H_, D_ = (int(v) for v in name.split(":")[1].split(","))
        c = dict(kind="stacked", batch=B_, seq=T_, hidden=H_, depth=D_)
    else:
        c = ftgen.CONFIGS[name]
    ws = ft.Workspace()
    if c["kind"] == "grid":
        g = ftgen.grid_inputs(c["batch"], c["len_x"], c["len_y"], c["hidden"], c["depth"], 1, "bf16")
        a = [torch.from_numpy(g[k]).cuda().to(torch.bfloat16) for k in ("x","ys","W","U")] + [torch.from_numpy(g["b"]).cuda()]
        fn = lambda: ft.grid_rnn(*a, workspace=ws)
    else:
        p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
        a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x","W","U")] + [torch.from_numpy(p["b"]).cuda()]
        dil = list(c.get("dilations", [])) or None
        fn = lambda: ft.stacked_lstm(*a, dilations=dil, workspace=ws)
    for _ in range(3): fn()
    buf = (ctypes.c_ulonglong * (1024 * 16))()
    L.ft_debug_trace(buf, 1024 * 16, 1)
    reps = 5
    for _ in range(reps): fn()
    torch.cuda.synchronize()
    L.ft_debug_trace(buf, 1024 * 16, 1)
    arr = np.array(buf[:], dtype=np.float64).reshape(1024, 16)[:148, :14] / reps
    tot = arr[:, 7].mean()
    print(name, "cycles/CTA/launch", f"{tot:.0f}", " tiles/CTA", arr[:, 8].mean())
    for i, n in [(k, NAMES[k]) for k in list(range(7)) + list(range(9, 14))]:
        even = arr[0::2, i].mean() / tot * 100; odd = arr[1::2, i].mean() / tot * 100
        print(f"  {n:9s} leader {even:5.1f}%  peer {odd:5.1f}%   max {arr[:, i].max()/tot*100:5.1f}%")
