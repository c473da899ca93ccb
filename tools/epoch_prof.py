"""Device timeline of one pipelined products epoch (diagnostic): torch.profiler (CUPTI) kernel
records, the union of their busy intervals against the epoch's span (idle = kernel-boundary
bubbles and host-bound stretches), and the count of gaps by size."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from synth.graphs import CONFIGS  # noqa: E402


def main():
    cfg = CONFIGS["products"]
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, Trainer
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg, torch.bfloat16)
    g = DeviceGraph(rp, col)
    kw = dict(feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16)
    _, _, C_ppm = B.clustering(g.g)
    t1 = Trainer(g, X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=1, k_max=1, sample_cache=False, **kw)
    est1 = t1.schedule(0)[2]
    del t1
    tr = Trainer(g, X, y, seeds, cfg.dims, cfg.fanout, cfg.F, Ws, bs, k_min=cfg.k_min, k_max=cfg.k_max,
                 mem_budget=int(est1[0]) // 8, C_ppm=C_ppm, pipeline=True, **kw)
    for e in range(3):
        tr.run_epoch(epoch=e, lr=0.01)
    torch.cuda.synchronize()
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        tr.run_epoch(epoch=3, lr=0.01)
        torch.cuda.synchronize()
    ev = [e for e in prof.events() if e.device_type.name == "CUDA"]
    iv = sorted((e.time_range.start, e.time_range.end) for e in ev)
    t0, t1_ = iv[0][0], max(e for _, e in iv)
    busy, cur_s, cur_e, gaps = 0, iv[0][0], iv[0][1], []
    for s, e in iv[1:]:
        if s > cur_e:
            busy += cur_e - cur_s
            gaps.append(s - cur_e)
            cur_s, cur_e = s, e
        else:
            cur_e = max(cur_e, e)
    busy += cur_e - cur_s
    span = t1_ - t0
    print(f"kernels/copies {len(iv)}; span {span / 1e3:.2f} ms; busy (union) {busy / 1e3:.2f} ms; "
          f"idle {(span - busy) / 1e3:.2f} ms in {len(gaps)} gaps")
    for lo, hi in ((0, 2), (2, 5), (5, 20), (20, 100), (100, 10 ** 9)):
        sel = [x for x in gaps if lo <= x < hi]
        print(f"  gaps {lo}-{hi} us: {len(sel)}, {sum(sel) / 1e3:.2f} ms")


if __name__ == "__main__":
    main()
