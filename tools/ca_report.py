"""Shared-memory traffic per MMA: ncu measurements vs the closed forms (DESIGN.md
"CA claim").  Reads gpurun_out/ca/*.csv written by
tools/ca_smem.sh and writes profiles/<round>/ca_smem.json + .md.

Per entry, bytes of SMEM traffic (writes + reads), normalised to one
"4096-flop MMA" (m16n8k16-equivalent) so schedules with different MMA shapes
compare:
    bytes_per_mma = (ld_bytes + st_bytes) / (2 m n k / 4096) / entries
Closed forms (kernel totals per entry, R20):
    1D  p kn s_e                2D  sqrt(p) (mk+kn) s_e
    3D  cbrt(p)(mk+kn) s_e + 2 (cbrt(p)-1) mn s_acc
    non-CA W_m x W_n warps: (mk+kn) s_e + (W_n mk + W_m kn) s_e
"""
import csv
import glob
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# tag -> (dtype, size, algo, p, batch, (Wm, Wn) for non-CA)
CASES = {}
for s, b in ((32, 8192), (64, 4096)):
    CASES[f"f64-{s}_1d"] = ("f64", s, "1d", {32: 2, 64: 8}[s], b)
    CASES[f"f64-{s}_2d"] = ("f64", s, "2d", {32: 4, 64: 16}[s], b)
    CASES[f"f64-{s}_3d"] = ("f64", s, "3d", 8, b)
    CASES[f"f64-{s}_nonca"] = ("f64", s, "nonca", 4, b)
CASES["f64-64_1dm8"] = ("f64", 64, "1d", 8, 4096)
CASES["f64-64_nonca16"] = ("f64", 64, "nonca", 16, 4096)
CASES["f64-64_nonca8"] = ("f64", 64, "nonca", 8, 4096)
CASES["f64-32_nonca8"] = ("f64", 32, "nonca", 8, 8192)
CASES["f16-64_nonca8"] = ("f16", 64, "nonca", 8, 8192)
CASES["f16-128_nonca16"] = ("f16", 128, "nonca", 16, 4096)
CASES["f16-64_w1d"] = ("f16", 64, "1d", 4, 8192)
CASES["f16-64_2d"] = ("f16", 64, "2d", 4, 8192)
CASES["f16-64_3d"] = ("f16", 64, "3d", 8, 8192)
CASES["f16-64_nonca"] = ("f16", 64, "nonca", 4, 8192)
CASES["f16-32_w1d"] = ("f16", 32, "1d", 2, 8192)
CASES["f16-32_2d"] = ("f16", 32, "2d", 4, 8192)
CASES["f16-32_nonca"] = ("f16", 32, "nonca", 4, 8192)
CASES["f16-128_w1d"] = ("f16", 128, "1d", 8, 4096)
CASES["f16-128_2d"] = ("f16", 128, "2d", 16, 4096)
CASES["f16-64_tc16"] = ("f16", 64, "tc16", 4, 8192)
CASES["f16-128_tc16"] = ("f16", 128, "tc16", 4, 4096)
# round 2: tcgen05 with A resident in TMEM (TS form), 1D and 3D k-layers
CASES["f16-64_ts1d"] = ("f16", 64, "tc16ts", 4, 8192)
CASES["f16-64_ts3d"] = ("f16", 64, "tc16ts", 8, 8192)
CASES["f16-128_ts1d"] = ("f16", 128, "tc16ts", 4, 4096)
CASES["f16-128_ts3d"] = ("f16", 128, "tc16ts", 8, 4096)
CASES["f16-32_ts1d"] = ("f16", 32, "tc16ts", 4, 8192)
CASES["f16-32_tc16"] = ("f16", 32, "tc16", 4, 8192)


def closed_form(dtype, s, algo, p):
    se = 8 if dtype == "f64" else 2
    sacc = 8 if dtype == "f64" else 4
    m = n = k = s
    if algo == "1d":
        return p * k * n * se
    if algo == "2d":
        return math.isqrt(p) * (m * k + k * n) * se
    if algo == "3d":
        c = round(p ** (1 / 3))
        # layer reduction: gather or reduce-scatter both move (c-1) partial
        # tiles through SMEM (write + read); reduce-scatter only balances it
        return c * (m * k + k * n) * se + 2 * (c - 1) * m * n * sacc
    if algo == "nonca":
        wm = {4: 2, 8: 4, 16: 4}[p]
        wn = p // wm
        return (m * k + k * n) * se + (wn * m * k + wm * k * n) * se
    if algo == "tc16":  # TMA writes A,B once; UMMA reads A,B once; epilogue stages C (write) + TMA store (read)
        return 2 * (m * k + k * n) * se + 2 * m * n * se
    if algo == "tc16ts":  # A: global -> registers -> TMEM (no SMEM); B: TMA write + UMMA read; C staged
        return 2 * k * n * se + 2 * m * n * se
    return None


def read(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Metric Name" in r)
    hdr = rows[h]
    mi, ui, vi = hdr.index("Metric Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "usecond": 1e3,
             "nsecond": 1, "msecond": 1e6}
    out = {}
    for r in rows[h + 1:]:
        try:
            out[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1)
        except ValueError:
            pass
    return out


def main(rnd="r1"):
    res = {}
    for f in sorted(glob.glob(os.path.join(ROOT, "gpurun_out", "ca", "*.csv"))):
        tag = os.path.basename(f)[:-4]
        if tag not in CASES:
            continue
        dtype, s, algo, p, batch = CASES[tag]
        d = read(f)
        ld = d.get("smsp__sass_data_bytes_mem_shared_op_ld.sum", 0)
        st = d.get("smsp__sass_data_bytes_mem_shared_op_st.sum", 0)
        tma_in = d.get("l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum", 0)
        tma_out = d.get("l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum", 0)
        mmas = 2.0 * s ** 3 / 4096 * batch
        per_entry = (ld + st) / batch
        if algo in ("tc16", "tc16ts"):  # async-proxy traffic is not LSU traffic: TMA bytes + analytic UMMA reads
            # (SS form: the tensor core reads A and B from SMEM once per entry; TS form: only B)
            umma_reads = (2 if algo == "tc16" else 1) * s * s * 2 * batch
            per_entry = (ld + st + tma_in + tma_out + umma_reads) / batch
        cf = closed_form(dtype, s, algo, p)
        wf_ld = d.get("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", 0)
        wf_st = d.get("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum", 0)
        bc = d.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", 0) + \
            d.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", 0)
        res[tag] = {"dtype": dtype, "size": s, "algo": algo, "p": p, "batch": batch,
                    "smem_ld_bytes": ld, "smem_st_bytes": st, "tma_ld_bytes": tma_in, "tma_st_bytes": tma_out,
                    "smem_bytes_per_entry": per_entry, "closed_form_bytes_per_entry": cf,
                    "smem_bytes_per_4096flop_mma": per_entry * batch / mmas,
                    "lsu_wavefronts": wf_ld + wf_st, "bank_conflicts": bc,
                    "theta": (1 - bc / (wf_ld + wf_st)) if (wf_ld + wf_st) else None,
                    "duration_ns": d.get("gpu__time_duration.sum")}
    outd = os.path.join(ROOT, "profiles", rnd)
    os.makedirs(outd, exist_ok=True)
    json.dump(res, open(os.path.join(outd, "ca_smem.json"), "w"), indent=1)
    lines = ["| case | SMEM B/entry (ncu) | closed form | B per 4096-flop MMA | bank conflicts | theta |",
             "|---|---|---|---|---|---|"]
    for tag, r in res.items():
        lines.append(f"| {tag} (p={r['p']}) | {r['smem_bytes_per_entry']:.0f} | {r['closed_form_bytes_per_entry']} | "
                     f"{r['smem_bytes_per_4096flop_mma']:.0f} | {r['bank_conflicts']:.0f} | "
                     f"{r['theta'] if r['theta'] is None else round(r['theta'], 4)} |")
    open(os.path.join(outd, "ca_smem.md"), "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main(*(sys.argv[1:]))
