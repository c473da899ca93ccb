"""Profiling driver: one arxiv-shaped Buffalo epoch (or a config given on the command line),
repeated, for ncu captures of individual kernels (not a benchmark; see bench.py)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from synth.graphs import CONFIGS  # noqa: E402
import bench  # noqa: E402


def main():
    cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "arxiv"]
    epochs = int(sys.argv[2]) if len(sys.argv) > 2 else 2
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import Trainer
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg)
    feats = X.to(torch.bfloat16).contiguous()
    tr = Trainer((rp, col), feats, y, seeds, cfg.dims,
                 cfg.fanout, cfg.F, Ws, bs, feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16,
                 k_min=cfg.k_min, k_max=max(cfg.k_min, min(cfg.k_max, 64)))
    if len(sys.argv) > 3 and sys.argv[3] == "auto":
        # bench.py's products calibration: M_ctr = Eq. 2 estimate of K=1 / 8
        t1 = Trainer((rp, col), feats, y, seeds, cfg.dims,
                     cfg.fanout, cfg.F, Ws, bs, feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16, k_min=1, k_max=1)
        _, _, est1, _ = t1.schedule(0)
        del t1
        tr.sched.mem_budget = int(est1[0]) // 8
    elif len(sys.argv) > 3:
        tr.sched.mem_budget = int(sys.argv[3])
    for e in range(epochs):
        st = tr.run_epoch(epoch=e, lr=0.01)
    torch.cuda.synchronize()
    print("K", st["K"], "edges", st["edges"], "groups", [g["n"] for g in st["groups"]])


if __name__ == "__main__":
    main()
