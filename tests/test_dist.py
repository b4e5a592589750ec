"""Multi-process host logic on CPU (gloo, world_size 2): photon-id sharding and
the int64 tally all-reduce give bit-identical tallies to the unsharded run
(SURVEY.md Sec. 8(e)).  The per-rank compute here is the oracle; on the GPU
box bench.py runs the same plumbing with libsr and NCCL."""
import os
import socket

import numpy as np
import pytest

import oracle
from paper_conf_cgo_damanijskymg20_b200 import inputs as I
from paper_conf_cgo_damanijskymg20_b200 import parallel as P

torch = pytest.importorskip("torch")

PER_RANK = 300


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _pack(o):
    return np.concatenate([o["A"].ravel(), o["Rd"], o["Tt"], o["counters_raw"]]).view(np.int64)


def _worker(rank, world, port, out_dir):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    off = P.task_offset_of(rank, PER_RANK)
    t = torch.from_numpy(_pack(oracle.mcml(p, off, PER_RANK, I.PRIMARY_SEED)).copy())
    P.allreduce_tallies(t)
    np.save(os.path.join(out_dir, f"r{rank}.npy"), t.numpy())
    dist.destroy_process_group()


def test_sharded_allreduce_is_bit_identical(tmp_path):
    import torch.multiprocessing as mp
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    m = I.C3
    p = oracle.mc_params(m.layers, m.n_above, m.n_below, m.dr, m.dz, m.nr, m.nz, m.step_cap)
    full = _pack(oracle.mcml(p, 0, world * PER_RANK, I.PRIMARY_SEED))
    for r in range(world):
        got = np.load(tmp_path / f"r{r}.npy")
        assert np.array_equal(got, full)


def test_split_even_covers_exactly():
    for total in (0, 1, 7, 1000, 10**9):
        for world in (1, 2, 3, 8):
            parts = [P.split_even(total, world, r) for r in range(world)]
            assert sum(c for _, c in parts) == total
            pos = 0
            for off, c in parts:
                assert off == pos
                pos += c
    assert P.task_offset_of(3, 10**7) == 3 * 10**7
    with pytest.raises(ValueError):
        P.task_offset_of(-1, 5)


def test_allreduce_without_process_group_is_identity():
    t = torch.arange(5, dtype=torch.int64)
    assert P.allreduce_tallies(t) is t
