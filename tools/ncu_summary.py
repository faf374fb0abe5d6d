"""Summarise an ncu --set full capture (.ncu-rep) and an ncu launch list (.csv) into profiles/.

    python tools/ncu_summary.py <rep.ncu-rep> <launches.csv> <tag> [flops_per_launch]
Writes profiles/<tag>_ncu_summary.json and profiles/<tag>_launches.csv.
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "lts__t_bytes.sum", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__ops_path_tensor_op_utchmma_src_bf16_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__inst_executed.sum",
]
SCALE = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "Tbyte": 1e12,
         "ms": 1e-3, "us": 1e-6, "ns": 1e-9, "s": 1.0}


def raw(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {}
        for h, u, v in zip(hdr, units, vals):
            d[h] = (v, u)
        res.append(d)
    return res


def num(v):
    try:
        return float(v.replace(",", ""))
    except ValueError:
        return None


def main():
    rep, launches, tag = sys.argv[1:4]
    flops = float(sys.argv[4]) if len(sys.argv) > 4 else None
    kernels = raw(rep)
    k = kernels[0]
    summ = {"source": os.path.basename(rep), "kernel": k.get("Kernel Name", ("?", ""))[0], "metrics": {}}
    for key in KEYS:
        if key in k:
            v, u = k[key]
            summ["metrics"][key] = {"value": num(v), "unit": u}
    m = summ["metrics"]
    rd = m["dram__bytes_read.sum"]["value"] * SCALE.get(m["dram__bytes_read.sum"]["unit"], 1)
    wr = m["dram__bytes_write.sum"]["value"] * SCALE.get(m["dram__bytes_write.sum"]["unit"], 1)
    t = m["gpu__time_duration.sum"]["value"] * SCALE.get(m["gpu__time_duration.sum"]["unit"], 1)
    summ["dram_bytes_per_launch"] = rd + wr
    summ["duration_s"] = t
    summ["dram_GBps"] = (rd + wr) / t / 1e9
    if flops:
        summ["flops_per_launch"] = flops
        summ["achieved_TFLOPs_under_ncu"] = flops / t / 1e12
    os.makedirs("profiles", exist_ok=True)
    with open(f"profiles/{tag}_ncu_summary.json", "w") as f:
        json.dump(summ, f, indent=1)
    if launches == "-":
        print(json.dumps(summ, indent=1))
        return
    # launch list: kernel name, count, mean duration, share
    rows = list(csv.reader(open(launches)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    agg = {}
    for r in rows[start + 1:]:
        if len(r) < len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d["Metric Name"] != "gpu__time_duration.sum":
            continue
        agg.setdefault(d["Kernel Name"], []).append(float(d["Metric Value"]))
    tot = sum(sum(v) for v in agg.values())
    with open(f"profiles/{tag}_launches.csv", "w") as f:
        f.write("kernel,launches,mean_ns,share_of_gpu_time\n")
        for name, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
            f.write(f"\"{name}\",{len(v)},{sum(v)/len(v):.0f},{sum(v)/tot:.4f}\n")
    print(json.dumps(summ, indent=1))


if __name__ == "__main__":
    main()
