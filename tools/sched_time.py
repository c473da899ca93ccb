"""Scheduler (buffalo_bucketize) timing per configuration (diagnostic): the K = 1 call (the
first statistics pass over every degree bucket + one group-size pass) against the calibrated
call (+ the micro-bucket passes of the explosion split + the K group-size passes)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from synth.graphs import CONFIGS  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "products"
    cfg = CONFIGS[name]
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, Trainer
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg, torch.bfloat16)
    g = DeviceGraph(rp, col)
    kw = dict(feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
    t1 = Trainer(g, X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=1, k_max=1, **kw)
    est1 = t1.schedule(0)[2]
    budget = int(est1[0]) // 8
    for label, k_lo, k_hi, b in (("K=1", 1, 1, (1 << 63) - 1), ("calibrated", cfg.k_min, cfg.k_max, budget)):
        tr = Trainer(g, X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=k_lo, k_max=k_hi, mem_budget=b, **kw)
        for e in range(2):
            tr.schedule(e)
        torch.cuda.synchronize()
        ts = []
        for e in range(2, 6):
            t = time.perf_counter()
            K = tr.schedule(e)[0]
            ts.append(1e3 * (time.perf_counter() - t))
        print(f"{name} {label}: K={K} k_tried={tr.plan.k_tried} items={tr.plan.num_items} "
              f"bucketize {min(ts):.2f} ms (min of 4), {sum(ts) / len(ts):.2f} mean", flush=True)
        del tr


if __name__ == "__main__":
    main()
