"""Multi-rank host logic on CPU: world_size-2 gloo processes shard regions, compute
their shard (oracle as the stand-in compute on CPU) and all-gather the results; the
gathered vector must equal the single-process result in global pair order."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_ipps_wangxc17_b200 import parallel, synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, regions_per_rank, q):
    import torch
    import torch.distributed as dist

    from oracle import core as oracle

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    r0, r1 = parallel.rank_regions(rank, world, regions_per_rank)
    b = synth.config_batch("C1", n_regions=r1 - r0, region_start=r0)
    local = torch.from_numpy(oracle.batch_log10(b))
    counts = [None] * world
    dist.all_gather_object(counts, int(local.numel()))
    n = max(counts)
    g = parallel.gather_results(parallel.pad_to(local, n), world)
    if rank == 0:
        q.put(parallel.unpad(g.numpy(), counts))
    dist.barrier()
    dist.destroy_process_group()


def test_rank_regions_partition():
    seen = []
    for r in range(4):
        a, b = parallel.rank_regions(r, 4, 5)
        seen += list(range(a, b))
    assert seen == list(range(20))
    with pytest.raises(ValueError):
        parallel.rank_regions(4, 4, 5)


def test_split_regions_balances_cells():
    cells = np.random.default_rng(0).integers(1, 100, size=1000)
    bnd = parallel.split_regions(1000, 8, cells)
    assert bnd[0] == 0 and bnd[-1] == 1000 and np.all(np.diff(bnd) > 0)
    per = [cells[bnd[i]:bnd[i + 1]].sum() for i in range(8)]
    assert max(per) - min(per) <= 2 * cells.max()


def test_gloo_world2_gather_equals_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, 1, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=180)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    from oracle import core as oracle

    ref = oracle.batch_log10(synth.config_batch("C1", n_regions=2, region_start=0))
    assert np.array_equal(got, ref)
