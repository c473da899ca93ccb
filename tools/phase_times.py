"""Phase breakdown of one Buffalo epoch with CUDA events (schedule / build / fwd / loss / bwd /
step), averaged over a few epochs after warm-up.  Diagnostic only; bench.py is the benchmark."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from synth.graphs import CONFIGS  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "arxiv"
    cfg = CONFIGS[name]
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import Trainer
    rp, col, X, y, seeds, Ws, bs = bench.make_inputs_device(cfg)
    feats = X.to(torch.bfloat16).contiguous()
    tr = Trainer((rp, col), feats, y, seeds, cfg.dims,
                 cfg.fanout, cfg.F, Ws, bs, feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16,
                 k_min=cfg.k_min, k_max=max(cfg.k_min, min(cfg.k_max, 64)))
    if name == "products":
        t2 = Trainer((rp, col), feats, y, seeds, cfg.dims,
                     cfg.fanout, cfg.F, Ws, bs, feat_dtype=B.BF16, gemm_mode=B.GEMM_BF16, k_min=1, k_max=1)
        _, _, est1, _ = t2.schedule(0)
        del t2
        tr.sched.mem_budget = int(est1[0]) // 8
    times = {}

    def ev():
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        return e

    def add(k, a, b):
        times[k] = times.get(k, 0.0) + a.elapsed_time(b)

    n_ep = 5
    for ep in range(n_ep + 2):
        torch.cuda.synchronize()
        w0 = time.perf_counter()
        e0 = ev()
        tr.loss.zero_()
        K, offs, est, ranks = tr.schedule(ep)
        e1 = ev()
        L = tr.L
        ea = ev()
        tr._ensure_arena(max(B.estimate_mem(tr.sizes_h[k, :L + 1], tr.sizes_h[k, L + 1:], tr.model)[0]
                             for k in range(K)))
        eb = ev()
        sampler = tr.sampler(ep)
        marks = []
        hb = hf = hk = 0.0
        for k in range(K):
            a = ev(); t0 = time.perf_counter()
            tr.build(offs[k], int(offs[k + 1] - offs[k]), sampler, tr.sizes_h[k]); t1 = time.perf_counter(); b = ev()
            tr.forward(); t2 = time.perf_counter(); c = ev()
            tr.loss_and_grad(offs[k], int(offs[k + 1] - offs[k])); d = ev()
            t3 = time.perf_counter(); tr.backward(); t4 = time.perf_counter(); e = ev()
            hb += t1 - t0; hf += t2 - t1; hk += t4 - t3
            marks.append((a, b, c, d, e))
        if ep >= 2:
            for nm, v in (("host build", hb), ("host fwd", hf), ("host bwd", hk)):
                times[nm] = times.get(nm, 0.0) + 1e3 * v
        s0 = ev(); tr.step(0.01); s1 = ev()
        torch.cuda.synchronize()
        wall = (time.perf_counter() - w0) * 1e3
        if ep >= 2:
            add("schedule", e0, e1)
            add("arena", ea, eb)
            for a, b, c, d, e in marks:
                add("build", a, b); add("fwd", b, c); add("loss", c, d); add("bwd", d, e)
            add("step", s0, s1)
            add("epoch(events)", e0, s1)
            times["epoch(wall)"] = times.get("epoch(wall)", 0.0) + wall
    for k, v in times.items():
        print(f"{k:16s} {v / n_ep:8.3f} ms")
    print("K", K)


if __name__ == "__main__":
    main()
