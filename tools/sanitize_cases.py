"""Small invocations of every kernel for compute-sanitizer (development aid)."""
import sys, os
import torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
dev = "cuda"
def run_seq(B, T, H, D, dt, dil=None, resident="1"):
    os.environ["FT_RESIDENT"] = resident
    p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16" if dt == torch.bfloat16 else "f32")
    a = [torch.from_numpy(p[k]).to(dev, dt) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).to(dev)]
    r = ft.stacked_lstm(*a, dilations=dil, want_all=True)
    torch.cuda.synchronize()
def run_grid(B, Lx, Ly, H, D, dt):
    g = ftgen.grid_inputs(B, Lx, Ly, H, D, 1, "bf16" if dt == torch.bfloat16 else "f32")
    a = [torch.from_numpy(g[k]).to(dev, dt) for k in ("x", "ys", "W", "U")] + [torch.from_numpy(g["b"]).to(dev)]
    ft.grid_rnn(*a, want_all=True)
    torch.cuda.synchronize()
run_seq(4, 5, 64, 2, torch.float32)
run_seq(5, 6, 128, 3, torch.bfloat16)                 # resident
run_seq(5, 6, 128, 3, torch.bfloat16, resident="0")   # streaming, 1 CTA
run_seq(130, 4, 128, 2, torch.bfloat16)               # streaming, CTA pair
run_seq(20, 7, 128, 3, torch.bfloat16, dil=[1, 2, 3])
run_grid(3, 3, 4, 64, 2, torch.bfloat16)
run_grid(3, 3, 4, 16, 2, torch.float32)
run_seq(256, 2, 1024, 5, torch.bfloat16, resident="0")  # streaming weights (80 MiB): persisting L2 window
os.environ["FT_TILE_UNITS"] = "32"
run_seq(130, 4, 128, 2, torch.bfloat16, resident="0")  # CTA pair, 32-unit tiles
os.environ.pop("FT_TILE_UNITS")
for band, owner, skew in (("2", "1", "1"), ("2", "0", "2"), ("3", "1", "2")):  # layer bands
    os.environ.update(FT_BAND=band, FT_OWNER=owner, FT_SKEW=skew)
    run_seq(256, 5, 128, 5, torch.bfloat16, resident="0")
    run_seq(100, 3, 128, 4, torch.bfloat16, resident="0")
for k in ("FT_BAND", "FT_OWNER", "FT_SKEW"):
    os.environ.pop(k)
p = ftgen.stacked_inputs(130, 4, 128, 2, 1, "bf16")       # NEXT-2 layer-sequential schedule
a = [torch.from_numpy(p[k]).to(dev, torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).to(dev)]
ft.stacked_lstm_layerwise(*a, want_all=True)
xs = torch.from_numpy(p["x"]).to(dev, torch.bfloat16)     # NEXT-3 linear RNN
ft.stacked_rnn(xs, a[1][:, 0].contiguous())
g = ftgen.b2b_inputs(256, 256, 64, 64, 1, "bf16")          # NEXT-4 back-to-back GEMMs
ft.b2b_gemm(*[torch.from_numpy(g[k]).to(dev, torch.bfloat16) for k in ("A", "B", "C")])
# round 2b features
os.environ["FT_CLUSTER"] = "1"                            # DSMEM cluster kernel (C2 class)
run_seq(37, 5, 128, 3, torch.bfloat16)
os.environ.pop("FT_CLUSTER")
run_seq(256, 6, 128, 6, torch.bfloat16, dil=[1, 2, 4, 1, 2, 4], resident="0")  # dilated, x read in place
os.environ["FT_OWNER_L0"] = "1"                           # layer-0 owners (dilated)
run_seq(256, 6, 128, 4, torch.bfloat16, dil=[1, 2, 3, 4], resident="0")
os.environ.pop("FT_OWNER_L0")
os.environ["FT_BAND"] = "2"                               # grid depth bands
run_grid(130, 3, 4, 128, 4, torch.bfloat16)
os.environ.update(FT_RESIDENT="0")                        # host-buffer call under bands (x/y overlap)
B, T, H, D = 256, 12, 128, 6
p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
W, U = (torch.from_numpy(p[k]).to(dev, torch.bfloat16) for k in ("W", "U"))
bb = torch.from_numpy(p["b"]).to(dev)
x_h = torch.from_numpy(p["x"]).to(torch.bfloat16).pin_memory()
y_h = torch.empty((B, T, H), dtype=torch.bfloat16).pin_memory()
hn_h = torch.empty((B, D, H), dtype=torch.bfloat16).pin_memory()
cn_h = torch.empty((B, D, H), dtype=torch.float32).pin_memory()
nb = ft.ft_stacked_lstm_hostio_workspace_size(B, T, H, D, ft.FT_BF16)
ws = torch.empty(nb, dtype=torch.uint8, device=dev)
s = torch.cuda.Stream()
ft.check(ft.ft_stacked_lstm_fwd_hostio(B, T, H, D, ft.FT_BF16, x_h.data_ptr(), W.data_ptr(), U.data_ptr(),
                                       bb.data_ptr(), y_h.data_ptr(), hn_h.data_ptr(), cn_h.data_ptr(),
                                       ws.data_ptr(), nb, s.cuda_stream))
s.synchronize()
os.environ.pop("FT_BAND")
# round 2 (this round) features
os.environ["FT_CLUSTER"] = "1"                            # cluster kernel, 16-unit slices (H = 128)
os.environ["FT_CLUSTER_UNITS"] = "16"
run_seq(40, 6, 128, 3, torch.bfloat16)
os.environ.pop("FT_CLUSTER_UNITS")
os.environ.pop("FT_CLUSTER")
os.environ["FT_BAND"] = "2"                               # SSA slot rings wrapping under bands
run_seq(256, 11, 64, 6, torch.bfloat16, resident="0")
os.environ.pop("FT_BAND")
run_seq(256, 11, 64, 4, torch.bfloat16, dil=[1, 2, 4, 3], resident="0")  # rings + layer-0 owners (default)
# last session of round 2: every layer owned (mode 3), 32-unit layer-0 slabs (<2,64,32>), recurrent half first
run_seq(256, 7, 512, 4, torch.bfloat16, dil=[1, 2, 4, 8], resident="0")
torch.cuda.synchronize()
print("sanitize cases done")
