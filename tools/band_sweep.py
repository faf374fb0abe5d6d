"""Sweep the KIND_SEQ wavefront order (layer bands, skew) and the weight L2 policy on one config.

usage: python tools/band_sweep.py CONFIG SETTING [SETTING ...]
  SETTING = comma list of ENV=VALUE (FT_BAND, FT_SKEW, FT_L2_RESIDENT_LAYERS, FT_L2_PERSIST_LAYERS,
            FT_TILE_UNITS) or "base".  Each setting is timed back to back (SW_REPS launches, power
            steady state) and its y / h_n / c_n are compared BITWISE with the default order (the
            per-cell arithmetic does not depend on the order).  Development aid; bench.py is the
            contract.
"""
import json, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)) + "/..")
import ftgen, bench
from paper_conf_sosp_liuqc0hs0y24_b200 import ft

KEYS = ("FT_BAND", "FT_SKEW", "FT_L2_RESIDENT_LAYERS", "FT_L2_PERSIST_LAYERS", "FT_TILE_UNITS", "FT_L2POL", "FT_DEBUG", "FT_OWNER", "FT_SPLIT_PHASE")


def main():
    name = sys.argv[1]
    if ":" in name:  # custom stacked spec  name:B,T,H,D
        B_, T_, H_, D_ = (int(v) for v in name.split(":")[1].split(","))
        c = dict(kind="stacked", batch=B_, seq=T_, hidden=H_, depth=D_)
    else:
        c = ftgen.CONFIGS[name]
    B, T, H, D = c["batch"], c["seq"], c["hidden"], c["depth"]
    p = ftgen.stacked_inputs(B, T, H, D, 1, "bf16")
    a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
    ws = ft.Workspace()
    flops = 16 * H * H * T * D * B
    reps = int(os.environ.get("SW_REPS", "150"))
    ref = None
    for setting in sys.argv[2:]:
        for k in KEYS:
            os.environ.pop(k, None)
        if setting != "base":
            for kv in setting.split(","):
                k, v = kv.split("=")
                os.environ[k] = v
        out = ft.stacked_lstm(*a, workspace=ws)
        torch.cuda.synchronize()
        outs = [out[k].clone() for k in ("y", "h_n", "c_n")]
        if ref is None and setting == "base":
            ref = outs
        same = None if ref is None else all(torch.equal(u, v) for u, v in zip(outs, ref))
        fn = lambda: ft.stacked_lstm(*a, workspace=ws)
        for _ in range(5):
            fn()
        torch.cuda.synchronize()
        cs = bench.ClockSampler(0)
        cs.start()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
        for s, e in ev:
            s.record(); fn(); e.record()
        torch.cuda.synchronize()
        clk = cs.stop() or {}
        ts = np.array([s.elapsed_time(e) for s, e in ev])
        med = float(np.median(ts[reps // 3:]))
        print(json.dumps(dict(cfg=name, setting=setting, ms_median=round(med, 4), ms_min=round(float(ts.min()), 4),
                              tflops=round(flops / med / 1e9, 1), bitwise_equal_default=same,
                              sm_mhz=clk.get("sm_mhz"), power_w=clk.get("power_w_median"))), flush=True)


if __name__ == "__main__":
    main()
