"""Step timeline of the layer-sequential recurrent kernel (CTA 0), from libft_trace.so."""
import ctypes, sys, os, json
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
ft.LIB_PATH = os.path.abspath("build/trace/libft_trace.so")
L = ft.lib()
for spec in sys.argv[1:] or ["256,100,1024,16", "32,100,1024,16"]:
    B, T, H, D = map(int, spec.split(","))
    p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
    a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
    ws = ft.Workspace()
    for _ in range(3): ft.stacked_lstm_layerwise(*a, workspace=ws)
    torch.cuda.synchronize()
    n = D * T
    buf = (ctypes.c_ulonglong * (n * 6))()
    L.ft_debug_lw_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
    L.ft_debug_lw_events(buf, n)
    ev = np.array(buf[:], dtype=np.float64).reshape(D, T, 6)
    e = ev[:, 2:T - 1]           # steady steps (t >= 2, t < T-1)
    prev_rel = ev[:, 1:T - 2, 5]
    out = dict(spec=spec,
               step_ns=float(np.median(np.diff(ev[:, 1:T - 1, 0], axis=1))),
               release_to_seen=float(np.median(e[..., 0] - prev_rel)),
               seen_to_first_A=float(np.median(e[..., 1] - e[..., 0])),
               first_A_to_last_mma=float(np.median(e[..., 2] - e[..., 1])),
               last_mma_to_tfull=float(np.median(e[..., 3] - e[..., 2])),
               tfull_to_stored=float(np.median(e[..., 4] - e[..., 3])),
               release_ns=float(np.median(e[..., 5] - e[..., 4])),
               layer_ns=[float(ev[d, T - 2, 5] - ev[d, 1, 0]) for d in range(min(D, 3))])
    print(json.dumps(out), flush=True)
