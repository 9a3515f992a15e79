"""Multi-rank host logic on CPU (gloo): bench.py's own shard / pack / gather / unpack
functions (paper_conf_ipps_wangxc17_b200/parallel.py) at world sizes 2 and 4, with the
oracle as the stand-in compute. The job's results gathered on rank 0 must equal the
single-process (N = 1) results bit for bit, in global pair order, for the strong split
of a fixed region set (cell-balanced, whole regions, rank-local generation)
and for the weak split."""
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


def _job(workload, world, rank, scaling, n_regions):
    """What one bench.py rank computes: its shard, its slot (oracle results)."""
    import torch

    from oracle import core as oracle

    r0, r1, pair_start, total_pairs, total_cells, cells = parallel.shard(workload, rank, world, scaling, n_regions)
    b = synth.config_batch(workload, n_regions=r1 - r0, region_start=r0)
    assert b.cells() == cells
    res = torch.from_numpy(oracle.batch_log10(b))
    return res, pair_start, total_pairs, cells


def _worker(rank, world, port, workload, scaling, n_regions, q):
    import torch
    import torch.distributed as dist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    res, pair_start, total_pairs, cells = _job(workload, world, rank, scaling, n_regions)
    nn = torch.tensor([res.numel()], dtype=torch.int64)
    dist.all_reduce(nn, op=dist.ReduceOp.MAX)
    slot = parallel.pack_slot(res, pair_start, int(nn.item()))
    g = parallel.gather_slots(slot, world)
    cc = torch.tensor([float(cells)], dtype=torch.float64)
    dist.all_reduce(cc)
    if rank == 0:
        q.put((parallel.unpack_global(g.numpy(), total_pairs), float(cc.item())))
    dist.barrier()
    dist.destroy_process_group()


def _run(world, workload, scaling, n_regions):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, workload, scaling, n_regions, q))
             for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    return got


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


@pytest.mark.parametrize("world", [2, 4, 8])
def test_full_c5_strong_split_is_cell_balanced(world):
    """The 2^26-pair C5 job (262,144 regions) split by cells: every rank within 0.01 % of
    total/world (whole regions of ~1.25e7 cells each), the shards tile the job."""
    spans = [parallel.shard("C5", r, world, "strong", 262144) for r in range(world)]
    total_pairs, total_cells = spans[0][3], spans[0][4]
    assert total_pairs == 1 << 26
    assert [s[0] for s in spans[1:]] == [s[1] for s in spans[:-1]] and spans[-1][1] == 262144
    assert [s[2] for s in spans] == list(np.cumsum([0] + [32 * 8 * (s[1] - s[0]) for s in spans[:-1]]))
    cells = np.array([s[5] for s in spans], dtype=np.float64)
    assert cells.sum() == total_cells
    assert np.max(np.abs(cells / (total_cells / world) - 1)) < 1e-4


def test_unpack_global_rejects_overlaps_and_gaps():
    g = np.array([[0, 2, 1.0, 2.0, np.nan], [2, 3, 3.0, 4.0, 5.0]])
    assert np.array_equal(parallel.unpack_global(g, 5), [1, 2, 3, 4, 5])
    with pytest.raises(ValueError):
        parallel.unpack_global(np.array([[0, 2, 1.0, 2.0, 0], [1, 3, 3.0, 4.0, 5.0]]), 5)
    with pytest.raises(ValueError):
        parallel.unpack_global(np.array([[0, 2, 1.0, 2.0, 0], [3, 2, 3.0, 4.0, 0]]), 5)


@pytest.mark.parametrize("world", [2, 4])
def test_gloo_strong_split_gather_is_bitwise_single_process(world):
    from oracle import core as oracle

    got, cells = _run(world, "C5", "strong", 12)
    ref = oracle.batch_log10(synth.config_batch("C5", n_regions=12))
    assert np.array_equal(got, ref)
    assert cells == synth.config_batch("C5", n_regions=12).cells()


@pytest.mark.parametrize("world", [2, 4])
def test_gloo_weak_split_gather_is_bitwise_single_process(world):
    from oracle import core as oracle

    got, _ = _run(world, "C1", "weak", 1)
    ref = oracle.batch_log10(synth.config_batch("C1", n_regions=world))
    assert np.array_equal(got, ref)
