"""Multi-process (gloo, world size 2, CPU) coverage of the N>1 host logic:
instance-range sharding and the additive CHECKSUM reduction are invariant
under the number of ranks (a multi-GPU run reproduces the
single-GPU output).  Keystreams come from the oracle; only the host-side
sharding/reduction code under test is shared with bench.py."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from helpers import checksum, to_sliced
from paper_conf_icppw_monfaredhkzrg20_b200 import inputs, shard

N_TOTAL, BITS = 32 * 6 + 7, 256


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        first, n = shard.strong_range(rank, world, N_TOTAL)
        keys, ivs = inputs.make_inputs("mickey2", n, first)
        rows = oracle.mickey2_keystream_batch(keys, ivs, 80, BITS, threads=1)
        local = checksum(to_sliced(rows), t0=0, g_base=first // 32)
        total = shard.allreduce_checksum(local)
        tmax = shard.allreduce_max(float(rank + 1))
        q.put((rank, first, n, total, tmax))
    finally:
        dist.destroy_process_group()


def _run(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out)


def test_strong_range_partition():
    for world in (1, 2, 3, 4, 8):
        for n_total in (1, 31, 32, 33, 1000, 1 << 20):
            spans = [shard.strong_range(r, world, n_total) for r in range(world)]
            assert sum(n for _, n in spans) == n_total
            pos = 0
            for first, n in spans:
                if n:
                    assert first == pos and first % 32 == 0
                    pos += n


def test_weak_range():
    assert shard.weak_range(3, 1 << 22) == (3 << 22, 1 << 22)
    with pytest.raises(ValueError):
        shard.weak_range(0, 33)


def test_int64_wrap():
    for u in (0, 1, (1 << 63) - 1, 1 << 63, (1 << 64) - 1):
        assert shard.to_int64(u) & shard.MASK64 == u


@pytest.mark.timeout(300)
def test_gloo_world2_checksum_is_shard_invariant():
    keys, ivs = inputs.make_inputs("mickey2", N_TOTAL)
    whole = checksum(to_sliced(oracle.mickey2_keystream_batch(keys, ivs, 80, BITS)))
    out = _run(2)
    assert [o[0] for o in out] == [0, 1]
    assert out[0][2] + out[1][2] == N_TOTAL
    assert out[0][3] == out[1][3] == whole
    assert out[0][4] == out[1][4] == 2.0
