"""Render a bf16_sweep.json (tools/bf16_sweep.py) as the markdown table in profiles/."""
import json
import statistics
import sys

src, dst = sys.argv[1], sys.argv[2]
d = json.load(open(src))
pts = d["points"] if isinstance(d, dict) and "points" in d else d
fr = [p["frac"] for p in pts]
lo = min(pts, key=lambda p: p["frac"])
with open(dst, "w") as f:
    f.write("# BF16 sweep (BASELINE configs[4]) — one B200, 125 000 entries per point (10^6 / 8 GPUs)\n\n")
    f.write("Each point: CUDA-event timing after warm-ups; `tools/bf16_sweep.py`. Run-to-run variance between "
            "boxes is up to ~10 % on individual points.\n\n")
    f.write(f"Summary: {len(pts)} points, roofline fraction median {statistics.median(fr):.3f}, "
            f"min {min(fr):.3f} ({lo['m']}x{lo['n']}x{lo['k']}), max {max(fr):.3f}.\n\n")
    f.write("| m | n | k | TFLOP/s | GB/s | frac of HBM roofline | kernel |\n|---|---|---|---|---|---|---|\n")
    for p in pts:
        f.write(f"| {p['m']} | {p['n']} | {p['k']} | {p['tflops']:.1f} | {p['gbs']:.0f} | {p['frac']:.3f} | "
                f"{p.get('kernel', '')} |\n")
