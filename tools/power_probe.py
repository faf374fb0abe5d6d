"""Power / clock behaviour of one workload run back to back for a few seconds (development aid).

    python tools/power_probe.py MODE [SECONDS]

MODE: gemm (torch bf16 8192^3 matmul, the MEASURED_PEAKS reference load) or a config name of
ftgen.CONFIGS (C2..C5).  Env FT_DEBUG etc. pass through to the library.  Prints one JSON line:
per-launch times over the run, and the nvidia-smi time series (SM clock, instantaneous and
averaged board power, throttle-reason bitmask) at 20 Hz, summarised per 0.5 s window.
"""
import json, os, subprocess, sys, tempfile, time
import numpy as np, torch

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)) + "/..")

FIELDS = "timestamp,clocks.sm,power.draw.instant,power.draw.average,clocks_event_reasons.active,temperature.gpu,utilization.gpu"


def make_fn(mode):
    if mode == "gemm":
        a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
        b = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
        return (lambda: torch.matmul(a, b)), 2 * 8192 ** 3
    import ftgen
    from paper_conf_sosp_liuqc0hs0y24_b200 import ft
    c = ftgen.CONFIGS[mode]
    ws = ft.Workspace()
    if c["kind"] == "grid":
        g = ftgen.grid_inputs(c["batch"], c["len_x"], c["len_y"], c["hidden"], c["depth"], 1, "bf16")
        a = [torch.from_numpy(g[k]).cuda().to(torch.bfloat16) for k in ("x", "ys", "W", "U")] + \
            [torch.from_numpy(g["b"]).cuda()]
        return (lambda: ft.grid_rnn(*a, workspace=ws)), \
            48 * c["hidden"] ** 2 * c["len_x"] * c["len_y"] * c["depth"] * c["batch"]
    p = ftgen.stacked_inputs(c["batch"], c["seq"], c["hidden"], c["depth"], 1, "bf16")
    a = [torch.from_numpy(p[k]).cuda().to(torch.bfloat16) for k in ("x", "W", "U")] + [torch.from_numpy(p["b"]).cuda()]
    dil = list(c.get("dilations", [])) or None
    H, T, D, B = c["hidden"], c["seq"], c["depth"], c["batch"]
    return (lambda: ft.stacked_lstm(*a, dilations=dil, workspace=ws)), 16 * H * H * T * D * B


def main():
    mode = sys.argv[1]
    secs = float(sys.argv[2]) if len(sys.argv) > 2 else 5.0
    fn, flops = make_fn(mode)
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    time.sleep(2.0)  # let the clock recover
    fd, path = tempfile.mkstemp(suffix=".csv")
    os.close(fd)
    smi = subprocess.Popen(["nvidia-smi", "-i", "0", f"--query-gpu={FIELDS}", "--format=csv,noheader,nounits",
                            "-lms", "50", "-f", path], stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
    time.sleep(0.5)
    evs = []
    t_start = time.time()
    memq, memp = None, []
    while time.time() - t_start < secs:
        if memq is None and time.time() - t_start > secs / 2:
            memq = subprocess.Popen(["nvidia-smi", "-i", "0", "-q", "-d", "POWER"], stdout=subprocess.PIPE,
                                    stderr=subprocess.DEVNULL, text=True)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record()
        evs.append((time.time() - t_start, s, e))
        if len(evs) % 20 == 0:
            torch.cuda.synchronize()
    torch.cuda.synchronize()
    time.sleep(0.3)
    smi.terminate(); smi.wait()
    if memq is not None:
        txt = memq.communicate()[0]
        sec = txt.split("GPU Memory Power Readings")[-1] if "GPU Memory Power Readings" in txt else ""
        for line in sec.splitlines()[:3]:
            if "Average Power Draw" in line:
                try:
                    memp.append(float(line.split(":")[1].split()[0]))
                except (ValueError, IndexError):
                    pass
    ms = [(t, s.elapsed_time(e)) for t, s, e in evs]
    rows = []
    for line in open(path):
        p = [x.strip() for x in line.split(",")]
        try:
            rows.append(dict(sm=float(p[1]), pi=float(p[2]), pa=float(p[3]), rs=int(p[4], 16), tmp=float(p[5]), util=float(p[6])))
        except (ValueError, IndexError):
            continue
    os.unlink(path)
    load = [r for r in rows if r["util"] > 50]
    arr = np.array([m for _, m in ms])
    nwin = max(1, int(secs / 0.5))
    wins = []
    for w in range(nwin):
        sel = [m for t, m in ms if w * 0.5 <= t < (w + 1) * 0.5]
        if sel:
            wins.append(round(float(np.median(sel)), 3))
    out = dict(mode=mode, ab=os.environ.get("FT_AB"), debug=os.environ.get("FT_DEBUG", "0"), launches=len(ms), ms_median=float(np.median(arr)),
               ms_min=float(arr.min()), ms_first=float(arr[0]), tflops_median=flops / np.median(arr) / 1e9,
               ms_per_halfsec=wins,
               sm_mhz=[r["sm"] for r in load], power_inst=[r["pi"] for r in load], power_avg=[r["pa"] for r in load],
               reasons=sorted({hex(r["rs"]) for r in load}), mem_power_w=memp, temp=[r["tmp"] for r in load][-1:] if load else None)
    for k in ("sm_mhz", "power_inst", "power_avg"):
        v = out[k]
        out[k + "_median"] = float(np.median(v)) if v else None
        out[k] = v[::4]  # thin the series
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
