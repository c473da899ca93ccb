"""The NCCL plumbing of the N > 1 path, executed on a B200 (the sandbox and the round-end tests
have one GPU, so the process group has one rank; NCCL refuses two ranks on one device).  The
collectives are the ones the trainer issues on a multi-GPU box (§V-G):
  * the scheduler's statistics all-gather — the library calls buffalo_sched.allgather, which
    buffalo.make_allgather implements with all_gather_into_tensor on device buffers;
  * the per-layer gradient all-reduce on a communication stream (train.allreduce_grads over
    slices of the flat gradient buffer, ordered after the producing stream by an event).
With one rank both are identities; the test checks they run through NCCL and return the data."""
import os
import socket
import subprocess
import sys
import textwrap

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = textwrap.dedent("""
    import ctypes, os, sys
    import numpy as np
    import torch
    import torch.distributed as dist
    sys.path.insert(0, {root!r})
    from paper_conf_hpca_yangzl25_b200 import buffalo as B
    from paper_conf_hpca_yangzl25_b200.train import allreduce_grads
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method="tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    assert dist.get_backend() == "nccl"
    # statistics all-gather through the library's callback type
    fn = B.make_allgather(1, dist.group.WORLD, torch.device("cuda", 0))
    send = (np.arange(1000, dtype=np.int64) * 7919) % 104729
    recv = np.zeros_like(send)
    rc = fn(None, send.ctypes.data, recv.ctypes.data, send.nbytes)
    assert rc == 0 and np.array_equal(recv, send), "all-gather callback"
    # per-layer gradient all-reduce on a comm stream after the producer
    g = torch.randn(206895, device="cuda")
    ref = g.clone()
    comm = torch.cuda.Stream()
    for a, b in ((100000, 206895), (40000, 100000), (0, 40000)):
        g[a:b].mul_(1.0)
        ev = torch.cuda.current_stream().record_event()
        comm.wait_event(ev)
        with torch.cuda.stream(comm):
            allreduce_grads(g[a:b], 2, dist.group.WORLD)   # world > 1 takes the collective path
    torch.cuda.current_stream().wait_stream(comm)
    torch.cuda.synchronize()
    assert torch.equal(g, ref), "all-reduce over one rank must return the data"
    dist.destroy_process_group()
    print("nccl ok")
""")


def test_nccl_collectives_execute():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    code = SCRIPT.format(root=ROOT, port=port)
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=300,
                       env=dict(os.environ, NCCL_DEBUG="WARN"))
    assert r.returncode == 0 and "nccl ok" in r.stdout, (r.stdout + r.stderr)[-3000:]
