"""Model vs measurement for every candidate schedule of the BASELINE configs
(profiles/r2/variant_sweep_r2.json) -> profiles/r2/planner_model_r2.md.
CPU only (the planner's model needs no device)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402
from test_planner_model import family, measured_for_plan  # noqa: E402

sw = json.load(open(os.path.join(ROOT, "profiles", "r2", "variant_sweep_r2.json")))
out = ["# Planner model vs measured (round 2)", "",
       "AUTO = argmax of the B200 cycle model (planner.cpp) over every schedule the library can run for the",
       "shape; measured = tools/variant_sweep_r2.py on one B200 (CUDA-graph timing).  `pick` marks AUTO's",
       "schedule; `best` the measured-fastest.  tests/test_planner_model.py asserts pick >= 0.95 best.", "",
       "| config | schedule | measured TF/s | model TF/s | model bound | |", "|---|---|---|---|---|---|"]
for cfg in sw["configs"]:
    dt, m, n, k = cfg["dtype"], cfg["m"], cfg["n"], cfg["k"]
    plan = kami.plan(m, n, k, dt)
    model = {(c["kernel"], c["algo"], c["p"]): c for c in kami.plan_candidates(m, n, k, dt)}
    best = max(c["tflops"] for c in cfg["candidates"] if c["algo"] != "auto")
    got = measured_for_plan(cfg, plan)
    for c in cfg["candidates"]:
        if c["algo"] == "auto":
            continue
        f = family(c["kernel"])
        mc = None
        for (kk, a, p), v in model.items():
            if kk == f and (a == c["algo"] or (f in ("tcgen05", "dmma_gen") and c["algo"] == "1d")
                            or (f == "dmma_tma" and c["algo"] == "1d_tma")) and \
                    (f != "warp_ca" or p == c["p"] or (c["p"] == 0 and a != "1d")):
                mc = v
        tag = []
        if got is not None and abs(c["tflops"] - got) < 1e-9:
            tag.append("pick")
        if c["tflops"] == best:
            tag.append("best")
        out.append(f"| {cfg['cfg']} | {c['kernel']} ({c['algo']}, p={c['p']}) | {c['tflops']:.1f} | "
                   f"{mc['model_tflops']:.1f} | {mc['bound']} | {' '.join(tag)} |" if mc else
                   f"| {cfg['cfg']} | {c['kernel']} ({c['algo']}, p={c['p']}) | {c['tflops']:.1f} | - | - | "
                   f"{' '.join(tag)} |")
open(os.path.join(ROOT, "profiles", "r2", "planner_model_r2.md"), "w").write("\n".join(out) + "\n")
print("\n".join(out))
