"""Shared helpers of the GPU parity tests: run the CUDA path through the C ABI and read its
outputs back.  The expected values come only from oracle/ (never from the CUDA path)."""
import numpy as np
import torch

from paper_conf_hpca_yangzl25_b200 import build_lib

build_lib.build()
from paper_conf_hpca_yangzl25_b200 import buffalo as B  # noqa: E402
from paper_conf_hpca_yangzl25_b200.train import DeviceGraph, Trainer  # noqa: E402


def arena_view(arena, p, n, dtype=torch.int32):
    if not p or n == 0:
        return torch.zeros(0, dtype=dtype)
    es = torch.empty(0, dtype=dtype).element_size()
    off = p - arena.data_ptr()
    assert off % es == 0 and off >= 0
    return arena.view(dtype)[off // es: off // es + n]


def blocks_to_numpy(arena, blocks, L):
    out = []
    for l in range(1, L + 1):
        b = blocks.layer[l - 1]
        d = dict(n_dst=b.n_dst, n_src=b.n_src, n_edges=b.n_edges, n_heavy=b.n_heavy)
        d["row_ptr"] = arena_view(arena, b.row_ptr, b.n_dst + 1).cpu().numpy()
        d["col_local"] = arena_view(arena, b.col_local, b.n_edges).cpu().numpy()
        d["src_global"] = arena_view(arena, b.src_global, b.n_src).cpu().numpy()
        d["col_global"] = arena_view(arena, b.col_global, b.n_edges).cpu().numpy() if b.col_global else None
        d["t_row_ptr"] = arena_view(arena, b.t_row_ptr, b.n_src + 1).cpu().numpy() if b.t_row_ptr else None
        d["t_col"] = arena_view(arena, b.t_col, b.n_edges).cpu().numpy() if b.t_col else None
        d["heavy"] = arena_view(arena, b.heavy, b.n_heavy).cpu().numpy() if b.heavy else None
        d["cls_perm"] = arena_view(arena, b.cls_perm, b.n_dst).cpu().numpy()
        d["t_perm"] = arena_view(arena, b.t_perm, b.n_src).cpu().numpy() if b.t_perm else None
        d["n_heavy_t"] = b.n_heavy_t
        out.append(d)
    return out


def act_view(arena, p, n, ld, dtype):
    t = arena_view(arena, p, n * ld, dtype)
    return t.view(n, ld).float().cpu().numpy()


def make_trainer(rp, col, X, y, seeds, dims, fanout, F, Ws, bs, gemm=B.GEMM_FFMA, feat_dtype=B.FP32, **kw):
    dev = "cuda"
    tdtype = torch.float32 if feat_dtype == B.FP32 else torch.bfloat16
    pitch = B.pitch(dims[0])
    Xp = np.zeros((X.shape[0], pitch), np.float32)
    Xp[:, :X.shape[1]] = X[:, :dims[0]]
    feats = torch.as_tensor(Xp).to(dev).to(tdtype).contiguous()
    labels = torch.as_tensor(np.asarray(y, np.int32)).to(dev)
    sd = torch.as_tensor(np.asarray(seeds, np.int32)).to(dev)
    return Trainer((rp, col), feats, labels, sd, dims, fanout, F, Ws, bs, feat_dtype=feat_dtype,
                   gemm_mode=gemm, **kw)


def close(gpu, ref, rtol, atol):
    gpu = np.asarray(gpu, np.float64)
    ref = np.asarray(ref, np.float64)
    err = np.abs(gpu - ref)
    bad = err > atol + rtol * np.abs(ref)
    return (not bad.any()), float(err.max() if err.size else 0.0), int(bad.sum())


def assert_close(gpu, ref, rtol, atol, what=""):
    ok, mx, nbad = close(gpu, ref, rtol, atol)
    assert ok, f"{what}: {nbad} elements out of tolerance (max abs err {mx:g})"


def assert_bf16_close(gpu, ref, what="", rel=2e-2):
    """Appendix C rule for the bf16-GEMM path: |gpu - ref| <= rel*|ref| + rel*rms(ref)."""
    ref = np.asarray(ref, np.float64)
    rms = float(np.sqrt(np.mean(ref ** 2))) if ref.size else 0.0
    assert_close(gpu, ref, rel, rel * rms + 1e-6, what)


def assert_normwise(gpu, ref, rel, what=""):
    """Reduced-precision gradients: ||gpu - ref||_F <= rel * ||ref||_F (ReLU masks of bf16
    activations may flip on near-zero pre-activations, so elementwise bounds do not apply)."""
    gpu = np.asarray(gpu, np.float64)
    ref = np.asarray(ref, np.float64)
    num = float(np.linalg.norm(gpu - ref))
    den = float(np.linalg.norm(ref))
    assert num <= rel * den + 1e-12, f"{what}: normwise rel error {num / max(den, 1e-30):.3g} > {rel}"
