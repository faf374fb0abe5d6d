"""Host-side cost of one forward call (development aid): wall time per call of the raw C-ABI entry
point (ctypes, preallocated buffers) issued back to back without synchronising, for C2 and C3
shapes.  The GPU runs asynchronously, so for launch-bound shapes this is the serving-loop
overhead the library adds (tensor maps, occupancy and attributes are cached after the first
call; the first call is reported separately)."""
import sys
import time
import torch
sys.path.insert(0, ".")
import ftgen  # noqa: E402
from paper_conf_sosp_liuqc0hs0y24_b200 import ft  # noqa: E402

for name in sys.argv[1:] or ["C2", "C3"]:
    c = ftgen.CONFIGS[name]
    B, T, H, D = c["batch"], c["seq"], c["hidden"], c["depth"]
    p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
    x, W, U = (torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U"))
    b = torch.from_numpy(p["b"]).cuda()
    y = torch.empty((B, T, H), dtype=torch.bfloat16, device="cuda")
    hn = torch.empty((B, D, H), dtype=torch.bfloat16, device="cuda")
    cn = torch.empty((B, D, H), dtype=torch.float32, device="cuda")
    nb = ft.ft_stacked_lstm_workspace_size(B, T, H, D, ft.FT_BF16, 0)
    ws = torch.empty(nb, dtype=torch.uint8, device="cuda")
    sp = torch.cuda.current_stream().cuda_stream
    args = (B, T, H, D, ft.FT_BF16, x.data_ptr(), W.data_ptr(), U.data_ptr(), b.data_ptr(), y.data_ptr(),
            hn.data_ptr(), cn.data_ptr(), None, None, ws.data_ptr(), nb, sp)
    t0 = time.perf_counter()
    ft.check(ft.ft_stacked_lstm_fwd(*args))
    first = time.perf_counter() - t0
    torch.cuda.synchronize()
    n = 50
    t0 = time.perf_counter()
    for _ in range(n):
        ft.check(ft.ft_stacked_lstm_fwd(*args))
    host = (time.perf_counter() - t0) / n
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        ft.check(ft.ft_stacked_lstm_fwd(*args))
    e1.record()
    torch.cuda.synchronize()
    print(f"{name}: first call {first * 1e6:.0f} us host; steady {host * 1e6:.1f} us host per call; "
          f"device {e0.elapsed_time(e1) / n * 1e3:.1f} us per forward")
