"""Sustained-load timing of one tcgen05 workload under KAMI_TC_TUNE variants
(each in its own process; the knob is read once per process).

    python tools/tc_tune.py --workload f16-64 --tunes "0,0,0,-1" "4,0,0,-1" ...
"""
import argparse
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(workload, reps):
    sys.path.insert(0, ROOT)
    import torch
    import kami_inputs as ki
    import paper_conf_sc_wangdltsl25_b200 as kami
    from bench import parse_workload, op_bytes
    dtype, m, n, k, batch, _ = parse_workload(workload)
    A, B = ki.operands(m, n, k, batch, dtype, "unif", device="cuda")
    C = torch.empty(batch * m * n, dtype=ki.TORCH_DTYPES[ki.OUT_DTYPE[dtype]], device="cuda")
    f = lambda: kami.gemm_strided_batched(m, n, k, batch, dtype, "row", A, B, C)  # noqa: E731
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    t_end = time.time() + 1.0
    while time.time() < t_end:
        for _ in range(10):
            f()
        torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for s, e in ev:
        s.record()
        f()
        e.record()
    torch.cuda.synchronize()
    ts = sorted(s.elapsed_time(e) for s, e in ev)
    t = ts[len(ts) // 2] * 1e-3
    print(json.dumps({"us": t * 1e6, "GBs": batch * op_bytes(dtype, m, n, k) / t / 1e9,
                      "TF": 2 * m * n * k * batch / t / 1e12}))


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="f16-64")
    ap.add_argument("--tunes", nargs="+", default=["0,0,0,-1"])
    ap.add_argument("--reps", type=int, default=30)
    ap.add_argument("--child", action="store_true")
    a = ap.parse_args()
    if a.child:
        child(a.workload, a.reps)
        sys.exit(0)
    for t in a.tunes:
        env = dict(os.environ, KAMI_TC_TUNE=t)
        r = subprocess.run([sys.executable, __file__, "--child", "--workload", a.workload, "--reps", str(a.reps)],
                           env=env, capture_output=True, text=True, timeout=300)
        print(a.workload, t, r.stdout.strip() or r.stderr[-500:], flush=True)
