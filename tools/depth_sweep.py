"""Fig. 8 protocol on this build: forward time vs depth for the
one-launch wavefront and for the same stacked LSTM run layer by layer (one launch per layer, the
'DAG approach' of Fig. 2 / L67).  The paper's hypothesis (L415): with maximal exploitable
parallelism the time grows sub-linearly with depth.  Writes JSON lines."""
import sys, json
import torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft

def timeit(fn, reps=10):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps

B = 256
for H in (256, 1024):
    for T in (32, 64, 128):
        p = ftgen.stacked_inputs(B, T, H, 32, 7, "bf16")
        x = torch.from_numpy(p["x"]).cuda().to(torch.bfloat16)
        W = torch.from_numpy(p["W"]).cuda().to(torch.bfloat16)
        U = torch.from_numpy(p["U"]).cuda().to(torch.bfloat16)
        b = torch.from_numpy(p["b"]).cuda()
        ws = ft.Workspace()
        for D in (1, 4, 8, 12, 16, 20, 24, 28, 32):
            wf = timeit(lambda: ft.stacked_lstm(x, W[:D], U[:D], b[:D], workspace=ws))
            def per_layer():
                inp = x
                for d in range(D):
                    r = ft.stacked_lstm(inp, W[d:d + 1], U[d:d + 1], b[d:d + 1], workspace=ws, want_all=True)
                    inp = r["h_all"][:, 0]
                return inp
            pl = timeit(per_layer, reps=3) if (D <= 16 or H == 256) else None
            print(json.dumps(dict(H=H, T=T, D=D, wavefront_ms=wf, per_layer_ms=pl)), flush=True)
