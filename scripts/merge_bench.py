"""Microbench of the exchange merge on one GPU (diagnostic, not a bench.py value):
P runs of (u32 key, u32 val), each sorted, as one rank receives them after the C5
key-range all-to-all, merged by rw_merge_runs (columns in) and by rw_pack_tuples +
rw_merge_packed_runs.  Prints ms and the effective GB/s of one read + one write of
the data (the single-pass design's algorithmic bytes)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_wudcy12_b200 import dist as rd  # noqa: E402


def main():
    P = int(os.environ.get("P", 8))
    n = int(os.environ.get("ROWS", 3 << 27)) // P
    dev = "cuda:0"
    g = torch.Generator(device=dev).manual_seed(5)
    keys, vals = [], []
    for _ in range(P):
        k = torch.randint(0, 1 << 30, (n,), device=dev, generator=g, dtype=torch.int64)
        v = torch.randint(0, 1 << 30, (n,), device=dev, generator=g, dtype=torch.int64)
        kv, _ = torch.sort(k * (1 << 31) + v)
        keys.append((kv >> 31).to(torch.int32))
        vals.append((kv & ((1 << 31) - 1)).to(torch.int32))
    cols = [torch.cat(keys), torch.cat(vals)]
    del keys, vals
    run_off = [i * n for i in range(P + 1)]
    be = rd.GpuBackend(0)
    types = ["u32", "u32"]
    out = {}
    packed = be.pack(cols, types)
    for name, fn in (("cols", lambda: be.merge(cols, types, run_off)),
                     ("packed", lambda: be.merge_packed(packed, types, run_off))):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        reps = 10
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        byts = P * n * 8 * 2
        out[name] = {"ms": round(ms, 4), "GBps_one_pass": round(byts / ms / 1e6, 1)}
    res = be.merge_packed(packed, types, run_off)
    ok = bool(torch.all(res[0][1:].to(torch.int64) >= res[0][:-1].to(torch.int64)).item())
    print(json.dumps({"P": P, "rows": P * n, "sorted": ok, **out}))


if __name__ == "__main__":
    main()
