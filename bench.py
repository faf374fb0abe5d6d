#!/usr/bin/env python
"""bench.py — stacked-LSTM wavefront throughput on B200 (the BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--gather fused|nccl|none]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...
(`--gpus N > 1` without torchrun launches the N ranks itself; it exits 2 if fewer than N GPUs are
visible, and a torchrun whose WORLD_SIZE differs from --gpus is refused the same way.)

Workload: BASELINE.json configs[2] ("C3"): stacked LSTM depth 16, seq 100, batch 256 per GPU,
hidden 1024, bf16 operands / fp32 accumulation — the configuration the metric is quoted on.
A step = one full forward of the nest (every cell of every diagonal) over one batch — one
ft_stacked_lstm_fwd call (flag reset + the persistent wavefront kernel).  Multi-GPU: the batch
`map` is sharded (each rank runs 256 sequences: weak scaling), no collective in the data path
except the north star's final output gather of y / h_n / c_n to rank 0, which is inside every
timed step: `fused` (default) maps rank 0's output buffers into every rank (the library's
ft_ipc_* calls: CUDA IPC / NVLink peer memory) so the kernel epilogue writes there directly
(SURVEY NEXT-1); `nccl` runs the library's ft_comm_gather_rank after each forward.  Afterwards
rank 0 recomputes every shard and checks the gathered outputs bitwise (`gather_ok`, pin P12).

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
    # torchrun exports OMP_NUM_THREADS=1; the CPU baseline uses every host core it may run on,
    # threads bound close.  Must run before the oracle library is first loaded
    # (OpenMP reads these at initialisation).
    os.environ["OMP_NUM_THREADS"] = str(host_cores())
    os.environ.setdefault("OMP_PROC_BIND", "close")
    os.environ.setdefault("OMP_PLACES", "cores" if host_info().get("threads_per_core", 1) == 1 else "threads")


def oracle_rate(p, rows, tsteps=None):
    """Time the CPU oracle (f32 instantiation of the unchanged source, built -O3 -march=native:
    oracle.build_timing) on `rows` batch rows of the workload, optionally only the first
    `tsteps` time steps.  Returns (seconds, sequences)."""
    import oracle
    x = p["x"][:rows] if tsteps is None else p["x"][:rows, :tsteps]
    t0 = time.perf_counter()
    oracle.stacked_lstm(x, p["W"], p["U"], p["b"], precision="f32", build_kind="timing")
    dt = time.perf_counter() - t0
    frac = 1.0 if tsteps is None else tsteps / p["x"].shape[1]
    return dt, rows * frac


def host_info():
    """The CPU the oracle baseline ran on: model, logical CPUs, affinity,
    sockets, cores per socket, threads per core (lscpu)."""
    info = {"cpu_model": None, "logical_cpus": os.cpu_count(), "affinity_cpus": None,
            "sockets": None, "cores_per_socket": None, "threads_per_core": None}
    try:
        info["affinity_cpus"] = len(os.sched_getaffinity(0))
    except AttributeError:
        pass
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            k, v = k.strip(), v.strip()
            if k == "Model name":
                info["cpu_model"] = v
            elif k == "Socket(s)":
                info["sockets"] = int(v)
            elif k == "Core(s) per socket":
                info["cores_per_socket"] = int(v)
            elif k == "Thread(s) per core":
                info["threads_per_core"] = int(v)
    except (OSError, ValueError, subprocess.SubprocessError):
        pass
    return info


def cpu_baseline(p):
    """the fp32 oracle (timing build), OpenMP over batch rows on every host
    core (bound close), 1 warm-up then the median of 3 runs on a bounded row sample."""
    info = host_info()  # before OpenMP binds this thread (the affinity mask shrinks then)
    pin_oracle_threads()
    import oracle
    n = oracle.num_threads("timing")
    oracle_rate(p, n)  # warm-up
    runs = [oracle_rate(p, n) for _ in range(3)]
    dt = statistics.median(r[0] for r in runs)
    seqs = runs[0][1]
    flop_per_seq = 16.0 * p["W"].shape[-1] ** 2 * p["x"].shape[1] * p["W"].shape[0]
    return dict({"value": seqs / dt, "unit": UNIT, "cores": n, "kind": "oracle",
                 "gflops": seqs * flop_per_seq / dt / 1e9,
                 "sample": f"{n} of 256 batch rows of C3 (full depth 16, seq 100; rows are independent "
                           f"by the batch map, P6), f32 instantiation of oracle/ft_oracle.c built -O3 "
                           f"-march=native -ffp-contract=off (bitwise the parity build), OpenMP over rows "
                           f"with OMP_PROC_BIND={os.environ.get('OMP_PROC_BIND')}; 1 warm-up, median of 3 "
                           f"runs = {dt:.2f} s (runs {', '.join(f'{r[0]:.2f}' for r in runs)} s)",
                 "protocol": "1 warm-up + median of 3"}, **info)


def bench_parity(p, got):
    """Achieved error of the benched forward (report it on the bench line): rows
    {0, B-1} of rank 0's batch through the fp64 oracle (rows are independent, P6), per output the
    normwise max|gpu-ref|/max|ref| (reading R19, tolerance 2e-2) and the RMS-relative error."""
    import numpy as np
    import oracle
    rows = [0, p["x"].shape[0] - 1]
    t0 = time.perf_counter()
    ref = oracle.stacked_lstm(p["x"][rows], p["W"], p["U"], p["b"], precision="f64", build_kind="timing")
    out = {"rows": rows, "tol_normwise": 2e-2, "oracle": "f64 (oracle/ft_oracle.c)"}
    ok = True
    for k in ("y", "h_n", "c_n"):
        g = got[k][rows].float().cpu().numpy().astype(np.float64)
        r = ref[k]
        nw = float(np.max(np.abs(g - r)) / max(np.max(np.abs(r)), 1e-30))
        rr = float(np.sqrt(np.sum((g - r) ** 2)) / max(np.sqrt(np.sum(r * r)), 1e-30))
        out[k] = {"normwise_rel": nw, "rms_rel": rr}
        ok = ok and nw <= 2e-2
    out["pass"] = ok
    out["oracle_s"] = time.perf_counter() - t0
    return out


# ----------------------------------------------------------------------------- inputs
def make_x(rank):
    """x of rank `rank`'s shard: rows [rank*B, (rank+1)*B) of the global batch (the generator is
    counter-based, so any shard regenerates on its own)."""
    import ftgen
    c = ftgen.CONFIGS[WORKLOAD]
    seed = ftgen.config_seed(WORKLOAD)
    B, T, H = c["batch"], c["seq"], c["hidden"]
    n = B * T * H
    return ftgen.round_bf16(ftgen.uniform(seed, ftgen.S_X, n, offset=rank * n).reshape(B, T, H))


def make_inputs(rank):
    import ftgen
    c = ftgen.CONFIGS[WORKLOAD]
    seed = ftgen.config_seed(WORKLOAD)
    H, D = c["hidden"], c["depth"]
    p = ftgen.stacked_inputs(1, 1, H, D, seed, "bf16")  # W, U, b (replicated on every rank)
    p["x"] = make_x(rank)
    return c, p


def shared_gpu_mode():
    """FT_BENCH_SHARED_GPU=1: every rank runs on cuda:0 (the 1-GPU tests of the N-rank path:
    gloo control plane, fused gather over CUDA IPC within one device)."""
    return os.environ.get("FT_BENCH_SHARED_GPU", "0") not in ("", "0")


# ----------------------------------------------------------------------------- reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    info = host_info()
    pin_oracle_threads()
    import oracle
    c, p = make_inputs(0)
    nthr = oracle.num_threads("timing")
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
    sample = (f"per step {nthr} of 256 C3 batch rows x first {tsteps} of {c['seq']} time steps (oracle "
              f"f32, -O3 -march=native timing build) "
              f"(work scales linearly in T; value counts {tsteps}/{c['seq']} of a sequence per row)")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": total / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": workload_config(1),
        "cpu_baseline": dict({"value": value, "unit": UNIT, "cores": nthr, "kind": "oracle",
                              "sample": sample}, **info),
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
    if world != args.gpus:
        # never report a rank count other than --gpus (main() self-launches N ranks when
        # WORLD_SIZE is unset, so this only trips on a mismatched external torchrun)
        print(f"error: WORLD_SIZE={world} != --gpus {args.gpus}", file=sys.stderr)
        return 2
    n_gpus = world
    shared = shared_gpu_mode()
    ndev = torch.cuda.device_count()
    if not shared and ndev < world:
        print(f"error: --gpus {world} needs {world} visible CUDA devices, found {ndev}", file=sys.stderr)
        return 2
    local = 0 if shared else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    # control plane: NCCL on distinct GPUs; gloo when the ranks share one GPU (the 1-GPU tests:
    # NCCL refuses two ranks on one device)
    backend = "gloo" if shared else os.environ.get("FT_DIST_BACKEND", "nccl")
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    gather = args.gather if args.gather is not None else ("fused" if world > 1 else "none")
    if world == 1:
        gather = "none"
    if gather == "nccl" and shared:
        print("error: --gather nccl needs one GPU per rank (FT_BENCH_SHARED_GPU is set)", file=sys.stderr)
        return 2

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
    from paper_conf_sosp_liuqc0hs0y24_b200.shard import CommGather, PeerGather
    gat = None
    gather_fallback = None
    if gather == "fused":
        # NEXT-1: y / h_n / c_n stored by the kernel epilogue straight into rank 0's buffers
        # (peer memory mapped by the library's ft_ipc_* calls; NVLink on an NVSwitch node)
        gat = PeerGather(B * world, T, H, D, bf, dev, dst=0)
        if not gat.ok():  # every rank agrees; fall back to the library's NCCL gather
            gather_fallback = f"fused gather unavailable ({gat.error or 'on another rank'}); used nccl"
            gat.close()
            gat, gather = None, ("nccl" if not shared else "none")
    if gather == "nccl":
        # the library's own NCCL gather (ft_comm_gather_rank), rank 0 in place
        gat = CommGather(B * world, T, H, D, bf, dev, dst=0)
        if not gat.ok():
            gather_fallback = (gather_fallback or "") + f"; nccl gather unavailable ({gat.error or 'on another rank'})"
            gat.close()
            gat, gather = None, "none"
    if gat is not None:
        outs = gat.local()
    stream = torch.cuda.current_stream()

    def step():
        ft.stacked_lstm(x, W, U, b, workspace=ws, out=outs)
        if gather == "nccl":  # the final output gather of y / h_n / c_n to rank 0 (NCCL)
            gat.gather(outs, stream.cuda_stream)
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.3)
    for _ in range(args.warmup):
        step()
    launch_desc = ft.ft_last_launch()  # the kernel + schedule the library picked for this step
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

    # the gathered outputs (P12): rank 0 recomputes every shard of the global batch on its own
    # GPU (same kernel, same 256-row shape, so per-row arithmetic is identical) and compares it
    # bitwise with what the gather delivered
    ref_local = ft.stacked_lstm(x, W, U, b, workspace=ws)
    gather_ok = None
    if gat is not None:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        if rank == 0:
            from paper_conf_sosp_liuqc0hs0y24_b200.shard import shard_rows
            gather_ok = True
            for r in range(world):
                a_, b_ = shard_rows(B * world, world, r)
                ref = ref_local if r == 0 else ft.stacked_lstm(
                    torch.from_numpy(make_x(r)).to(dev, bf), W, U, b, workspace=ws)
                for k in ("y", "h_n", "c_n"):
                    gather_ok = gather_ok and bool(torch.equal(gat.full[k][a_:b_], ref[k]))
        gat.close()

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
        ok = bool(torch.equal(y_h.to(dev), ref_local["y"]))
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
    parity = None if args.no_parity else bench_parity(p, ref_local)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": n_gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
        "data": "synthetic (ftgen splitmix64: x~U(-1,1), W,U,b~U(+-1/sqrt(H)), bf16 RNE)",
        "config": dict(workload_config(n_gpus), gather=gather,
                       gather_note={"none": "no output gather",
                                    "fused": "y/h_n/c_n stored by every rank's kernel epilogue into "
                                             "rank 0's buffers (peer memory, ft_ipc_*), inside the "
                                             "timed step",
                                    "nccl": "ft_comm_gather_rank (NCCL send/recv to rank 0) of "
                                            "y/h_n/c_n after each forward, inside the timed step"}[gather],
                       control_plane=backend if world > 1 else None,
                       ranks_share_one_gpu=bool(shared) if world > 1 else None),
        "gather_ok": gather_ok,
        "gather_fallback": gather_fallback,
        "parity": parity,
        "tensor_pipe_pct_of_peak": 100.0 * roofline["frac"],
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
        "gpu_launches": args.steps, "clocks": clocks,
        "kernels_per_step": {launch_desc: 1},
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
    ap.add_argument("--gather", default=None, choices=["none", "nccl", "fused"],
                    help="final output gather of y/h_n/c_n to rank 0, inside every timed step (N > 1; "
                         "default fused): fused = each rank's kernel epilogue stores into rank 0's "
                         "buffers over peer memory / NVLink (NEXT-1); nccl = the library's "
                         "ft_comm_gather_rank after each forward; none = no gather")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-parity", action="store_true",
                    help="skip the achieved-error check of the timed path on two sampled rows")
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return self_launch(args)
    return run_ours(args)


def self_launch(args):
    """`bench.py --gpus N` without torchrun: launch the N ranks ourselves (one process per GPU,
    torch.distributed.run on 127.0.0.1) and return their exit status.  Refuses (exit 2) when
    fewer than N devices are visible, so a run is never mislabelled with the wrong n_gpus."""
    import socket
    import torch
    ndev = torch.cuda.device_count()
    if not shared_gpu_mode() and ndev < args.gpus:
        print(f"error: --gpus {args.gpus} needs {args.gpus} visible CUDA devices, found {ndev}",
              file=sys.stderr)
        return 2
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    env = dict(os.environ)
    # NCCL's communicator lines (rank / nranks per communicator) on stderr-visible INFO output
    # (stderr, so rank 0's JSON line stays the only line on stdout)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    env.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd, env=env)


if __name__ == "__main__":
    sys.exit(main())
