"""The paper's block-level experiment on B200 (Sec. 5.1, Sec. 5.2,
Fig. 8/9/15): 16 384 entries launched at once, each team
loops the CA schedule `reps` times on chip (no global I/O in the loop).
Reports TFLOP/s per (dtype, order, schedule) and the measured per-entry cycle
breakdown (communication vs computation, clock64) next to the B200 cost model
(planner constants: L_sm 29, B_sm 127.6, O_tc 31.9 / 477 flop/cycle).

    python tools/block_level.py [--reps 1000] [--entries 16384] [--out profiles/r1/block_level.json]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402

CASES = [("f64", s, a, 0) for s in (16, 32, 64) for a in ("1d", "2d", "3d", "nonca")]
CASES += [("f16", 32, "1d", 2), ("f16", 32, "2d", 0), ("f16", 32, "nonca", 0)]
CASES += [("f16", 64, "1d", 4), ("f16", 64, "2d", 0), ("f16", 64, "3d", 0), ("f16", 64, "nonca", 0),
          ("f16", 64, "nonca", 8)]
CASES += [("f16", 128, "1d", 8), ("f16", 128, "2d", 0), ("f16", 128, "nonca", 16)]


def model(dtype, s, algo, p):
    if algo == "nonca":
        return None
    se = 8 if dtype == "f64" else 2
    O = 31.9 if dtype == "f64" else 477.0
    V, Tcm, Tcp, Tall = kami.paper_cost(algo, s, s, s, p, se, 29.0, 127.6, 1.0, 1.0, O, 4.0)
    stages = {"1d": p, "2d": round(p ** 0.5), "3d": round(p ** (1 / 3))}[algo]
    return {"stages": stages, "T_cm_per_stage": Tcm, "T_cp_per_warp_stage": Tcp, "T_all_paper": Tall,
            "comm_cycles_per_rep_model": stages * Tcm, "comp_cycles_per_rep_model": stages * Tcp * max(1.0, p / 4.0)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=1000)
    ap.add_argument("--entries", type=int, default=16384)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r1", "block_level.json"))
    a = ap.parse_args()
    res = []
    for dtype, s, algo, p in CASES:
        plan = kami.plan(s, s, s, dtype, algo=algo, p=p) if p or algo != "1d" or dtype == "f64" else None
        pp = p or (plan["p"] if plan else 0)
        A, B = ki.operands(s, s, s, a.entries, dtype, "unif", seed=0, device="cuda")
        C = torch.empty(a.entries * s * s, dtype=A.dtype, device="cuda")
        kami.gemm_block_level(s, s, s, a.entries, dtype, "row", A, B, C, algo=algo, p=pp, reps=2)  # warm
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        kami.gemm_block_level(s, s, s, a.entries, dtype, "row", A, B, C, algo=algo, p=pp, reps=a.reps)
        e1.record()
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) * 1e-3
        tf = 2.0 * s ** 3 * a.entries * a.reps / t / 1e12
        # cycle breakdown on a small launch (one entry per team, few teams per SM)
        nb = 148
        cyc = torch.zeros(2 * nb, dtype=torch.int64, device="cuda")
        kami.gemm_block_level(s, s, s, nb, dtype, "row", A, B, C, algo=algo, p=pp, reps=100, cycles=cyc)
        torch.cuda.synchronize()
        cy = cyc.view(nb, 2).double().mean(0) / pp / 100  # per warp per rep
        r = {"dtype": dtype, "order": s, "algo": algo, "p": pp, "entries": a.entries, "reps": a.reps,
             "tflops": tf, "ms": t * 1e3, "kernel": kami.last_kernel(),
             "comm_cycles_per_warp_rep": float(cy[0]), "comp_issue_cycles_per_warp_rep": float(cy[1]),
             "model": model(dtype, s, algo, pp)}
        res.append(r)
        print(json.dumps(r), flush=True)
        del A, B, C
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(res, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
