"""Host logic of bench.py's world-sim with shared statistics (--sim-shared): the all-gathers of
N simulated ranks are recorded call by call (record_allgathers) and replayed to each rank in turn
(AllgatherReplay).  A fake deterministic "scheduler" stands in for buffalo_bucketize: rank r's
rows at call i depend on r, i and everything gathered before (as the K loop's next statistics
pass depends on the previous ones), and the number of calls depends on the gathered data.  The
replay must hand every rank exactly what a real all-gather would, and refuse a rank whose own
rows differ from the recording."""
import ctypes

import numpy as np

import bench


def _fake_rank(r, world, fn, log=None):
    """Rank r's computation: up to 6 all-gathers of 5 int64 rows each; stops when the gathered
    sum crosses a threshold (a data-dependent call count, like Alg. 3's K loop)."""
    hist = 0
    for i in range(6):
        send = np.array([(r + 1) * 1000 + i * 10 + k + hist % 97 for k in range(5)], np.int64)
        recv = np.zeros(world * 5, np.int64)
        rc = fn(None, send.ctypes.data, recv.ctypes.data, send.nbytes)
        if rc != 0:
            return False
        if log is not None:
            log.append(recv.copy())
        hist += int(recv.sum())
        if hist > 40000:
            break
    return True


def _true_gathers(world):
    """The all-gather results of a lock-step run of all ranks (the ground truth)."""
    out, hist = [], 0
    for i in range(6):
        rows = [np.array([(r + 1) * 1000 + i * 10 + k + hist % 97 for k in range(5)], np.int64)
                for r in range(world)]
        g = np.concatenate(rows)
        out.append(g)
        hist += int(g.sum())
        if hist > 40000:
            break
    return out


def test_record_then_replay_matches_a_real_allgather():
    for world in (2, 3, 8):
        rep = bench.AllgatherReplay(world)
        rec = bench.record_allgathers(rep, lambda r: _fake_rank(r, world, rep.fn))
        truth = _true_gathers(world)
        assert len(rec) == len(truth)
        for a, b in zip(rec, truth):
            assert np.array_equal(np.frombuffer(a, np.int64), b)
        for r in range(world):                       # timed phase: each rank alone, replayed
            rep.rank, rep.results, rep.i = r, rec, 0
            log = []
            assert _fake_rank(r, world, rep.fn, log)
            assert rep.i == len(rec)
            assert all(np.array_equal(x, y) for x, y in zip(log, truth))


def test_replay_refuses_mismatched_rows():
    world = 2
    rep = bench.AllgatherReplay(world)
    rec = bench.record_allgathers(rep, lambda r: _fake_rank(r, world, rep.fn))
    rep.rank, rep.results, rep.i = 1, rec, 0
    bad = np.arange(5, dtype=np.int64)               # not rank 1's rows at call 0
    recv = np.zeros(world * 5, np.int64)
    assert rep.fn(None, bad.ctypes.data, recv.ctypes.data, bad.nbytes) == 1
    assert not recv.any()
