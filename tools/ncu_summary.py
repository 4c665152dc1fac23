"""Summarise ncu reports into profiles/<round>/ncu_summary.json.

    python tools/ncu_summary.py --round r1 --rep gpurun_out/r1/x.ncu-rep:f16-64 [...]
                                [--launches gpurun_out/r1/launches.csv]

For each report (one kernel launch, `ncu --set full`) records duration, DRAM
bytes (the `traffic` of bench.py's roofline object), throughput percentages,
tensor-pipe activity, shared-memory wavefronts / bank conflicts, registers and
occupancy.  For a launch list (`--metrics gpu__time_duration.sum`) records
each kernel's share of the summed device time.
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import defaultdict

KEYS = {
    "duration_ns": "gpu__time_duration.sum",
    "dram_read_bytes": "dram__bytes_read.sum",
    "dram_write_bytes": "dram__bytes_write.sum",
    "dram_throughput_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm_throughput_pct": "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "tensor_pipe_active_pct": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "smem_ld_wavefronts": "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
    "smem_st_wavefronts": "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
    "smem_ld_bytes": "smsp__sass_data_bytes_mem_shared_op_ld.sum",
    "smem_st_bytes": "smsp__sass_data_bytes_mem_shared_op_st.sum",
    "smem_ld_bank_conflicts": "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
    "smem_st_bank_conflicts": "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
    "tma_load_bytes": "l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum",
    "tma_store_bytes": "l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum",
    "registers_per_thread": "launch__registers_per_thread",
    "achieved_occupancy_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm_clock_hz": "smsp__cycles_elapsed.avg.per_second",
    "inst_executed": "smsp__inst_executed.sum",
    "dmma_inst": "smsp__inst_executed_pipe_fp64.sum",
}

UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "usecond": 1e3, "msecond": 1e6,
              "ns": 1, "us": 1e3, "ms": 1e6, "Ghz": 1e9, "Mhz": 1e6, "hz": 1, "cycle/nsecond": 1e9,
              "cycle/usecond": 1e6, "cycle/second": 1}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {}
        for h, u, v in zip(hdr, units, vals):
            d[h] = (u, v)
        res.append(d)
    return res


def num(u, v):
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return v
    return x * UNIT_SCALE.get(u, 1)


def summarise(rep):
    out = []
    for d in raw(rep):
        s = {"kernel": d.get("Kernel Name", ("", ""))[1][:120]}
        for k, m in KEYS.items():
            if m in d:
                s[k] = num(*d[m])
        if "dram_read_bytes" in s and "dram_write_bytes" in s:
            s["dram_bytes"] = s["dram_read_bytes"] + s["dram_write_bytes"]
        out.append(s)
    return out


def launches(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg = defaultdict(list)
    for r in rows[h + 1:]:
        agg[r[ki][:100]].append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in agg.values()) or 1.0
    return [{"kernel": k, "launches": len(v), "sum_ns": sum(v), "share": sum(v) / tot, "mean_ns": sum(v) / len(v)}
            for k, v in sorted(agg.items(), key=lambda x: -sum(x[1]))]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", required=True)
    ap.add_argument("--rep", action="append", default=[], help="path.ncu-rep:workload")
    ap.add_argument("--launches", action="append", default=[], help="path.csv:label")
    a = ap.parse_args()
    d = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", a.round)
    os.makedirs(d, exist_ok=True)
    f = os.path.join(d, "ncu_summary.json")
    summ = json.load(open(f)) if os.path.exists(f) else {"reports": {}, "launch_lists": {}, "traffic_bytes_per_launch": {}}
    for spec in a.rep:
        rep, _, wl = spec.rpartition(":")
        s = summarise(rep)
        summ["reports"][wl] = s
        if s and "dram_bytes" in s[0]:
            summ["traffic_bytes_per_launch"][wl] = s[0]["dram_bytes"]
    for spec in a.launches:
        p, _, label = spec.rpartition(":")
        summ["launch_lists"][label] = launches(p)
    json.dump(summ, open(f, "w"), indent=1)
    print(json.dumps(summ, indent=1)[:3000])


if __name__ == "__main__":
    main()
