"""Device timeline of one calibrated scheduler call (diagnostic): torch.profiler (CUPTI) kernel and
memcpy/memset records of buffalo_bucketize, in order, with the gaps between them — unlike an ncu
launch list this is not serialised or cache-flushed."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from synth.graphs import CONFIGS  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "papers"
    cfg = CONFIGS[name]
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, Trainer
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg, torch.bfloat16)
    g = DeviceGraph(rp, col)
    kw = dict(feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
    t1 = Trainer(g, X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=1, k_max=1, **kw)
    est1 = t1.schedule(0)[2]
    del t1
    tr = Trainer(g, X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=cfg.k_min, k_max=cfg.k_max,
                 mem_budget=int(est1[0]) // 8, **kw)
    for e in range(2):
        tr.schedule(e)
    torch.cuda.synchronize()
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        tr.schedule(2)
        torch.cuda.synchronize()
    ev = [e for e in prof.events() if e.device_type.name == "CUDA"]
    ev.sort(key=lambda e: e.time_range.start)
    t0 = ev[0].time_range.start
    prev_end = t0
    tot = {}
    for e in ev:
        s, d = e.time_range.start, e.time_range.end - e.time_range.start
        gap = s - prev_end
        prev_end = max(prev_end, e.time_range.end)
        nm = e.name.split("(")[0].replace("void buffalo::", "").replace("void ", "")[:48]
        tot[nm] = tot.get(nm, 0) + d
        print(f"{(s - t0) / 1e3:9.3f} ms  gap {gap / 1e3:7.3f}  {d / 1e3:8.3f} ms  {nm}")
    print(f"total span {(prev_end - t0) / 1e3:.3f} ms; busy {sum(tot.values()) / 1e3:.3f} ms")
    for k, v in sorted(tot.items(), key=lambda x: -x[1])[:12]:
        print(f"  {v / 1e3:8.3f} ms  {k}")


if __name__ == "__main__":
    main()
