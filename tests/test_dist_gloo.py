"""Multi-process (gloo, world_size 2, CPU) tests of the kernel-axis sharding and choice-table
all-gather (paper_conf_sc_fandccfc23_b200/dist.py).  The CUDA sweep is replaced by
the CPU oracle as a stand-in compute function (tests only); the shard / pad / gather / trim logic
is the product code."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_fandccfc23_b200.dist import ShardedSweep, shard_rows


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg, n_total, weak, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    models = W.make_models(cfg)
    sp, en, freqs, d = models
    targets = W.targets_six()

    def compute(feats, out):
        r = oracle.sweep(sp, en, feats.numpy(), freqs, d, targets)
        out.copy_(torch.from_numpy(r["choice"]))

    sh = ShardedSweep(n_total, len(targets), rank, world, torch.device("cpu"), compute=compute, weak=weak)
    feats = torch.from_numpy(W.make_features(cfg, sh.row0, sh.n_local))
    table = sh.run(feats)
    out_q.put((rank, table.numpy().copy(), sh.row0, sh.n_local))
    dist.barrier()
    dist.destroy_process_group()


def _run(cfg, n_total, weak, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, n_total, weak, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(res, key=lambda x: x[0])


def _reference(cfg, n_rows):
    import oracle
    from paper_conf_sc_fandccfc23_b200 import workloads as W
    sp, en, freqs, d = W.make_models(cfg)
    feats = W.make_features(cfg, 0, n_rows)
    return oracle.sweep(sp, en, feats, freqs, d, W.targets_six())["choice"]


def test_shard_rows_partition():
    for n in (0, 1, 5, 7, 16, 1001):
        for world in (1, 2, 3, 4, 8):
            seen = []
            for r in range(world):
                row0, cnt, per = shard_rows(n, r, world)
                assert cnt <= per and per == (n + world - 1) // world
                seen.extend(range(row0, row0 + cnt))
            assert seen == list(range(n))


@pytest.mark.parametrize("n_total", [16, 13])          # 13: uneven shards, padded last shard
def test_strong_scaling_gather_equals_single_process(n_total):
    res = _run("c1", n_total, weak=False)
    ref = _reference("c1", n_total)
    for rank, table, row0, n_local in res:
        assert table.shape == ref.shape
        np.testing.assert_array_equal(table, ref)          # every rank holds the full table


def test_weak_scaling_gather_concatenates_rank_populations():
    res = _run("c1", 6, weak=True)
    ref = _reference("c1", 12)                             # rank r sweeps rows [6r, 6r+6)
    for rank, table, row0, n_local in res:
        assert row0 == 6 * rank and n_local == 6
        np.testing.assert_array_equal(table, ref)
