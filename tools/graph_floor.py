"""Per-launch floor of graph-replayed kernels on this box (context for the
latency-bound configs[0]): K launches of a trivial torch kernel captured in
one CUDA graph, timed between two events, vs the same for the KAMI 16^3 x 1024
launch.  Not a product path."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402


def graph_time(fn, K=200):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(K):
            fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / K * 1e3  # us per launch


x = torch.zeros(1, device="cuda")
out = {"trivial_torch_add_us": graph_time(lambda: x.add_(1))}
A, B = ki.operands(16, 16, 16, 1024, "f16", "int", device="cuda")
C = torch.empty(1024 * 256, dtype=torch.float16, device="cuda")
out["kami_f16_16cubed_x1024_us"] = graph_time(
    lambda: kami.gemm_strided_batched(16, 16, 16, 1024, "f16", "row", A, B, C, stream=torch.cuda.current_stream()))
out["kernel"] = kami.last_kernel()
print(json.dumps(out))
