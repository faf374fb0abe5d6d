#!/usr/bin/env python
"""bench.py — stacked-LSTM wavefront throughput on B200 (the BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--gather]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...

Workload: BASELINE.json configs[2] ("C3"): stacked LSTM depth 16, seq 100, batch 256 per GPU,
hidden 1024, bf16 operands / fp32 accumulation — the configuration the metric is quoted on.
A step = one full forward of the nest (every cell of every diagonal) over one batch — one
ft_stacked_lstm_fwd call (flag reset + the persistent wavefront kernel).  Multi-GPU: the batch
`map` is sharded (each rank runs 256 sequences: weak scaling), no collective in the data path;
--gather [nccl|fused] adds the north star's final output gather of y to rank 0: `nccl` calls
torch.distributed.gather after each forward; `fused` maps rank 0's output buffers into every rank
(CUDA IPC / NVLink P2P) so the kernel epilogue writes there directly.

Prints ONE JSON line on rank 0.  Timing: W untimed warm-ups, then K steps bracketed by
barrier + cuda synchronize, CUDA events on the launching stream, max over ranks.  L2: the
inputs (268 MB of weights) exceed the 126 MB L2, no flush needed: the kernel runs the layers in
bands of 4 (67 MB of weights), so each step starts by loading band 0's weights from HBM again.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "stacked-LSTM sequences/sec (device-timed) at 1/2/4/8 B200; tensor-pipe % of peak"
UNIT = "sequences/s"
WORKLOAD = "C3"


def workload_config(n_gpus):
    import ftgen
    c = ftgen.CONFIGS[WORKLOAD]
    return {
        "workload": "C3: stacked LSTM depth=16, seq=100, batch=256 per GPU, hidden=1024, bf16 "
                    "(BASELINE.json configs[2])",
        "depth": c["depth"], "seq_len": c["seq"], "hidden": c["hidden"],
        "per_gpu_batch": c["batch"], "global_batch": c["batch"] * n_gpus,
        "parallelism": f"dp{n_gpus} (batch map sharded, weights replicated)",
        "l2": "inputs > L2 (268 MB of bf16 weights vs 126 MB L2), no flush: each step re-reads every "
              "layer band's weights from HBM (bands of 4 layers stay L2-resident only while they run)",
        "seed": ftgen.config_seed(WORKLOAD),
    }


def algorithmic_flops(c):
    # 2 * M * N * K per cell: M = batch, N = 4H, K = 2H (input + recurrent halves), every cell
    # (the t = 0 cells skip the zero recurrent half; counted as the paper's 16H^2 per cell-row)
    return 16.0 * c["hidden"] ** 2 * c["seq"] * c["depth"] * c["batch"]


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get("bf16_tflops"), d.get("bf16_tflops_sustained"), d.get("hbm_gbs"), "measured"
    return 1590.0, 1400.0, 6650.0, "fallback (B200_PROFILING.md)"


def load_traffic():
    """dram read+write bytes per launch from the committed ncu --set full summary, or None."""
    p = os.path.join(ROOT, "profiles", "latest_C3_ncu_summary.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get("dram_bytes_per_launch")
    return None


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("timestamp,clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap,utilization.gpu,power.draw.instant,power.limit")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.path = None

    def start(self):
        try:
            fd, self.path = tempfile.mkstemp(suffix=".csv")
            os.close(fd)
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50", "-f", self.path],
                stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    @staticmethod
    def _ts(text):
        # nvidia-smi timestamp "YYYY/MM/DD HH:MM:SS.mmm" (host local time) -> epoch seconds
        import datetime
        try:
            return datetime.datetime.strptime(text.strip(), "%Y/%m/%d %H:%M:%S.%f").timestamp()
        except ValueError:
            return None

    def stop(self, window=None):
        """Stop sampling; summarise the samples taken inside `window` = (t_start, t_end) host
        epoch seconds (the timed region) when there are any, else the samples under load."""
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        rows = []
        with open(self.path) as f:
            for line in f:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) < 10:
                    continue
                try:
                    rows.append(dict(ts=self._ts(parts[0]), sm=float(parts[1]), smax=float(parts[2]),
                                     hw=parts[3], hwt=parts[4], swt=parts[5], pc=parts[6],
                                     util=float(parts[7]), pw=float(parts[8]), plim=float(parts[9])))
                except ValueError:
                    continue
        os.unlink(self.path)
        if not rows:
            return None
        inside = []
        if window is not None:
            inside = [r for r in rows if r["ts"] is not None and window[0] - 0.02 <= r["ts"] <= window[1] + 0.02]
        loaded = inside or [r for r in rows if r["util"] > 50] or rows
        reasons = set()
        for r in loaded:
            for key, name in (("hw", "hw_slowdown"), ("hwt", "hw_thermal_slowdown"),
                              ("swt", "sw_thermal_slowdown"), ("pc", "sw_power_cap")):
                if r[key].lower().startswith("active"):
                    reasons.add(name)
        return {"sm_mhz": statistics.median(r["sm"] for r in loaded),
                "sm_max_mhz": max(r["smax"] for r in loaded), "reasons": sorted(reasons),
                # instantaneous board power (power.draw is a 1 s average and under-reads a
                # sub-second timed region); power.limit is the cap sw_power_cap enforces
                "power_w_median": statistics.median(r["pw"] for r in loaded),
                "power_limit_w": max(r["plim"] for r in loaded),
                "samples": len(loaded),
                "samples_from": "timed region" if inside else "samples under load (none inside the timed region)"}


# ----------------------------------------------------------------------------- CPU oracle
def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def load_ncu_tensor_pct():
    """ncu's tensor-pipe active % of the committed C3 capture (profiles/latest_C3_ncu_summary.json)."""
    try:
        with open(os.path.join(ROOT, "profiles", "latest_C3_ncu_summary.json")) as f:
            d = json.load(f)
        m = d.get("metrics", d)
        return m["sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"]["value"]
    except (OSError, KeyError, ValueError, TypeError):
        return None


def pin_oracle_threads():
    # torchrun exports OMP_NUM_THREADS=1; the CPU baseline uses every host core it may run on.
    # Must run before oracle/liboracle.so is first loaded (OpenMP reads it at initialisation).
    os.environ["OMP_NUM_THREADS"] = str(host_cores())


def oracle_rate(p, rows, tsteps=None):
    """Time the CPU oracle (f32 instantiation, as it stands) on `rows` batch rows of the
    workload, optionally only the first `tsteps` time steps.  Returns (seconds, sequences)."""
    import oracle
    x = p["x"][:rows] if tsteps is None else p["x"][:rows, :tsteps]
    t0 = time.perf_counter()
    oracle.stacked_lstm(x, p["W"], p["U"], p["b"], precision="f32")
    dt = time.perf_counter() - t0
    frac = 1.0 if tsteps is None else tsteps / p["x"].shape[1]
    return dt, rows * frac


def host_info():
    """The CPU the oracle baseline ran on: model, logical CPUs, affinity."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    try:
        aff = len(os.sched_getaffinity(0))
    except AttributeError:
        aff = None
    return {"cpu_model": model, "logical_cpus": os.cpu_count(), "affinity_cpus": aff}


def cpu_baseline(p):
    pin_oracle_threads()
    import oracle
    n = oracle.num_threads()
    dt, seqs = oracle_rate(p, n)
    flop_per_seq = 16.0 * p["W"].shape[-1] ** 2 * p["x"].shape[1] * p["W"].shape[0]
    return dict({"value": seqs / dt, "unit": UNIT, "cores": n, "kind": "oracle",
                 "gflops": seqs * flop_per_seq / dt / 1e9,
                 "sample": f"{n} of 256 batch rows of C3 (full depth 16, seq 100; rows are independent "
                           f"by the batch map, P6), f32 instantiation of oracle/ft_oracle.c, OpenMP over "
                           f"rows, {dt:.1f} s wall"}, **host_info())


# ----------------------------------------------------------------------------- inputs
def make_inputs(rank):
    import numpy as np
    import ftgen
    c = ftgen.CONFIGS[WORKLOAD]
    seed = ftgen.config_seed(WORKLOAD)
    B, T, H, D = c["batch"], c["seq"], c["hidden"], c["depth"]
    p = ftgen.stacked_inputs(1, 1, H, D, seed, "bf16")  # W, U, b (replicated on every rank)
    n = B * T * H  # this rank's rows [rank*B, (rank+1)*B) of the global batch
    p["x"] = ftgen.round_bf16(ftgen.uniform(seed, ftgen.S_X, n, offset=rank * n).reshape(B, T, H))
    return c, p


# ----------------------------------------------------------------------------- reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    pin_oracle_threads()
    import oracle
    c, p = make_inputs(0)
    nthr = oracle.num_threads()
    budget = float(os.environ.get("FT_REF_BUDGET_S", "150"))
    per_step = budget / max(1, args.steps + args.warmup)
    # calibrate: seconds per (row-parallel batch of nthr rows) per time step
    dt0, _ = oracle_rate(p, nthr, tsteps=2)
    per_t = dt0 / 2
    tsteps = int(max(1, min(c["seq"], per_step / max(per_t, 1e-9))))
    for _ in range(args.warmup):
        oracle_rate(p, nthr, tsteps)
    times, seqs = [], 0.0
    for _ in range(args.steps):
        dt, s = oracle_rate(p, nthr, tsteps)
        times.append(dt)
        seqs += s
    total = sum(times)
    value = seqs / total
    sample = (f"per step {nthr} of 256 C3 batch rows x first {tsteps} of {c['seq']} time steps "
              f"(work scales linearly in T; value counts {tsteps}/{c['seq']} of a sequence per row)")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": total / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": workload_config(1),
        "cpu_baseline": dict({"value": value, "unit": UNIT, "cores": nthr, "kind": "oracle",
                              "sample": sample}, **host_info()),
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------------------- our arm
def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_sosp_liuqc0hs0y24_b200 import ft

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus and world > 1:
        print(f"warning: WORLD_SIZE={world} != --gpus {args.gpus}", file=sys.stderr)
    n_gpus = world
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    backend = os.environ.get("FT_DIST_BACKEND", "nccl")  # gloo: exercise the multi-rank path on 1 GPU
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)

    def max_over_ranks(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    c, p = make_inputs(rank)
    B, T, H, D = c["batch"], c["seq"], c["hidden"], c["depth"]
    bf = torch.bfloat16
    x = torch.from_numpy(p["x"]).to(dev, bf)
    W = torch.from_numpy(p["W"]).to(dev, bf)
    U = torch.from_numpy(p["U"]).to(dev, bf)
    b = torch.from_numpy(p["b"]).to(dev)
    ws = ft.Workspace()
    outs = {"y": torch.empty((B, T, H), dtype=bf, device=dev),
            "h_n": torch.empty((B, D, H), dtype=bf, device=dev),
            "c_n": torch.empty((B, D, H), dtype=torch.float32, device=dev)}
    from paper_conf_sosp_liuqc0hs0y24_b200.shard import PeerGather, gather_rows
    if args.gather == "fused" and world > 1:
        # NEXT-1: y / h_n / c_n stored by the kernel epilogue straight into rank 0's buffers
        peer = PeerGather(B * world, T, H, D, bf, dev, dst=0)
        outs = peer.local()

    def step():
        ft.stacked_lstm(x, W, U, b, workspace=ws, out=outs)
        if args.gather == "nccl" and world > 1:  # the final output gather of y to rank 0 (NCCL)
            gather_rows(outs["y"], B * world, dst=0)

    stream = torch.cuda.current_stream()
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.3)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    host_t0 = time.time()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(stream)
    for i in range(args.steps):
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
    t1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    host_t1 = time.time()
    time.sleep(0.06)  # let the sampler write the sample that closes the window
    clocks = sampler.stop(window=(host_t0, host_t1))
    elapsed_ms = t0.elapsed_time(t1)
    call_ms = [s.elapsed_time(e) for s, e in ev]
    elapsed_ms = max_over_ranks(elapsed_ms)
    ms_per_step = elapsed_ms / args.steps
    value = n_gpus * B * args.steps / (elapsed_ms / 1e3)

    # roofline of the dominant kernel (the wavefront kernel is the whole step)
    peak_b, peak_s, hbm, peak_src = load_peaks()
    flops = algorithmic_flops(c)
    mean_call_s = statistics.mean(call_ms) / 1e3
    achieved = flops / mean_call_s / 1e12
    roofline = {"bound": "tensor", "achieved": achieved, "peak": peak_b, "unit": "TFLOP/s",
                "frac": achieved / peak_b, "traffic": load_traffic(),
                "peak_kind": f"{peak_src} dense bf16 burst (MEASURED_PEAKS.json bf16_tflops)",
                "frac_of_sustained": achieved / peak_s if peak_s else None,
                "flops_per_launch": flops,
                "launch_ms_mean": mean_call_s * 1e3,
                "note": "launch duration = one ft_stacked_lstm_fwd call: counter reset (memset) + the "
                        "persistent wavefront kernel, CUDA events on the launch stream",
                "launch_ms_median": statistics.median(call_ms), "launch_ms_min": min(call_ms)}
    # bound time of the binding roofline row (SURVEY d.2: tensor 4.26 ms, HBM 4.10 ms at C3) and
    # the DRAM side from the committed ncu capture
    t_tensor = flops / (peak_b * 1e12)
    roofline["t_bound_ms"] = t_tensor * 1e3
    tr = roofline["traffic"]
    if tr and hbm:
        roofline["hbm"] = {"bytes_per_launch_ncu": tr, "peak_GBps": hbm,
                           "frac": tr / mean_call_s / 1e9 / hbm}
    ncu_pct = load_ncu_tensor_pct()
    if ncu_pct is not None:
        roofline["ncu_tensor_pipe_active_pct"] = ncu_pct

    # the same achieved rate against the tensor peak at the clock the run actually had (148 SMs x
    # 8192 dense bf16 FLOP/clk/SM x the median SM clock sampled during the timed region): the
    # kernel's efficiency with the power cap's clock taken out
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    if clocks and clocks.get("sm_mhz"):
        clk_peak = nsm * 8192 * clocks["sm_mhz"] * 1e6 / 1e12
        roofline["clock_normalized"] = {"peak_at_sampled_clock_tflops": clk_peak,
                                        "frac": achieved / clk_peak,
                                        "sm_mhz": clocks["sm_mhz"]}

    # end to end through the public host-buffer C-ABI call (pinned host in/out, copies timed)
    e2e = None
    if True:  # every rank: its own shard through the host-buffer call; max over ranks below
        es = 2
        x_h = torch.from_numpy(p["x"]).to(bf).pin_memory()
        y_h = torch.empty((B, T, H), dtype=bf).pin_memory()
        hn_h = torch.empty((B, D, H), dtype=bf).pin_memory()
        cn_h = torch.empty((B, D, H), dtype=torch.float32).pin_memory()
        nb = ft.ft_stacked_lstm_hostio_workspace_size(B, T, H, D, ft.FT_BF16)
        wsh = torch.empty(nb, dtype=torch.uint8, device=dev)
        sp = stream.cuda_stream

        def e2e_step():
            ft.check(ft.ft_stacked_lstm_fwd_hostio(B, T, H, D, ft.FT_BF16, x_h.data_ptr(),
                                                   W.data_ptr(), U.data_ptr(), b.data_ptr(),
                                                   y_h.data_ptr(), hn_h.data_ptr(), cn_h.data_ptr(),
                                                   wsh.data_ptr(), nb, sp))
        ke = min(args.steps, 20)
        for _ in range(min(args.warmup, 3)):
            e2e_step()
        torch.cuda.synchronize()
        a0 = torch.cuda.Event(enable_timing=True)
        a1 = torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        for _ in range(ke):
            e2e_step()
        a1.record(stream)
        torch.cuda.synchronize()
        e_ms = max_over_ranks(a0.elapsed_time(a1))
        # sanity: the host result equals the device-path result of the same batch
        ok = bool(torch.equal(y_h.to(dev), outs["y"]))
        e2e = {"value": n_gpus * B * ke / (e_ms / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": B * T * H * es,
               "d2h_bytes_per_step": B * T * H * es + B * D * H * es + B * D * H * 4,
               "steps": ke, "api": "ft_stacked_lstm_fwd_hostio (pinned host buffers)",
               "matches_device_path": ok}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return 0
    cpu = None
    if n_gpus == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(p)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": n_gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
        "data": "synthetic (ftgen splitmix64: x~U(-1,1), W,U,b~U(+-1/sqrt(H)), bf16 RNE)",
        "config": dict(workload_config(n_gpus), gather=args.gather),
        "tensor_pipe_pct_of_peak": 100.0 * roofline["frac"],
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
        "gpu_launches": args.steps, "clocks": clocks,
        "kernels_per_step": {"wavefront_bf16_kernel<2, 64> (tcgen05/TMA, persistent; layer bands, "
                             "owner-computes; x read in place by 3-D TMA)": 1},
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=("ours", "reference"), default="ours")
    ap.add_argument("--gather", nargs="?", const="nccl", default="none", choices=["none", "nccl", "fused"],
                    help="gather y to rank 0 each step: nccl = torch.distributed.gather after the kernel; "
                         "fused = the kernel stores into rank 0's buffer over NVLink (NEXT-1)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
