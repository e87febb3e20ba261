"""N>1 host logic on CPU (-m "not gpu"): world_size-2 gloo process group.

Each rank takes its shard of the stimulus pairs at every operating point
(shard_pairs, as bench.py does; Context.set_pair_range), computes the
shard's activity / latest arrival (with the oracle standing in for the GPU),
and reduce_results() combines them on rank 0 -- exactly the bench.py path
with NCCL replaced by gloo.  Rank 0 checks the result equals the full run.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _shard_results(w, slots):
    import oracle
    P = w.stimuli.n_pairs
    V = len(w.vdd)
    r = oracle.simulate(w.netlist, w.library, w.stimuli, w.vdd, slots % P, slots // P, cap=64)
    act = np.zeros((w.netlist.n_signals, V), np.int64)
    lat = np.zeros(V, np.float32)
    for i, s in enumerate(slots):
        k = s // P
        act[:, k] += r.count[i]
        po = w.netlist.po_sig
        c = r.count[i, po]
        if (c > 0).any():
            last = r.times[i, po, np.maximum(c - 1, 0)][c > 0].max()
            lat[k] = max(lat[k], np.float32(last))
    return act, lat


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_date_schneiderw20_b200.parallel import shard_pairs, reduce_results
    from workloads import make_config
    w = make_config(3, n_pairs=40, n_vdd=3, scale=0.02)
    P, V = w.stimuli.n_pairs, len(w.vdd)
    first, n = shard_pairs(P, rank, world)
    act, lat = _shard_results(w, np.array([k * P + j for j in range(first, first + n) for k in range(V)]))
    ta, tl = torch.from_numpy(act), torch.from_numpy(lat)
    reduce_results(ta, tl, dst=0)
    if rank == 0:
        fa, fl = _shard_results(w, np.arange(w.n_slots))
        q.put((bool(np.array_equal(ta.numpy(), fa)), bool(np.array_equal(tl.numpy(), fl)), int(fa.sum())))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_shard_and_reduce():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    assert all(p.exitcode == 0 for p in procs)
    ok_act, ok_lat, total = q.get(timeout=5)
    assert ok_act and ok_lat and total > 0


@pytest.mark.parametrize("total,world", [(65536, 8), (96, 2), (7, 3), (1, 1)])
def test_shard_range_partitions(total, world):
    from paper_conf_date_schneiderw20_b200.parallel import shard_range
    spans = [shard_range(total, r, world) for r in range(world)]
    assert spans[0][0] == 0
    for (a, n), (b, _) in zip(spans, spans[1:]):
        assert a + n == b
    assert sum(n for _, n in spans) == total
    assert max(n for _, n in spans) - min(n for _, n in spans) <= 1
