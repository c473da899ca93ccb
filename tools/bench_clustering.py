"""Times the GPU triangle counting + C of Eq. 1 (buffalo_triangles / buffalo_avg_clustering) on a
BASELINE-shaped synthetic graph (diagnostic; prints one JSON line).
usage: python tools/bench_clustering.py [products|arxiv|...] [reps]"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_yangzl25_b200 import buffalo as B  # noqa: E402
from synth import device as SD  # noqa: E402
from synth.graphs import CONFIGS  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "products"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    cfg = CONFIGS[name]
    rp, col = SD.random_graph(cfg.N, cfg.pairs, cfg.kind)
    g = B.Graph()
    g.num_nodes, g.nnz, g.row_ptr, g.col = cfg.N, col.numel(), rp.data_ptr(), col.data_ptr()
    ws = torch.empty(B.clustering_workspace_bytes(g), dtype=torch.uint8, device="cuda")
    T = torch.empty(cfg.N, dtype=torch.int64, device="cuda")
    for _ in range(2):
        B.triangles(g, T, ws)
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    ms = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        B.triangles(g, T, ws)
        e1.record(s)
        e1.synchronize()
        ms.append(e0.elapsed_time(e1))
    C, ppm = B.avg_clustering(g, T, ws)
    d = (rp[1:] - rp[:-1]).double()
    wedges = float((d * (d - 1) / 2).sum())
    tri = int(T.sum().item()) // 3
    ms.sort()
    print(json.dumps({"graph": name, "N": cfg.N, "nnz": int(col.numel()), "triangles": tri, "wedges": wedges,
                      "C": C, "C_ppm": ppm, "ms_median": ms[len(ms) // 2], "ms_all": ms,
                      "edges_per_s": col.numel() / 2 / (ms[len(ms) // 2] * 1e-3)}))


if __name__ == "__main__":
    main()
