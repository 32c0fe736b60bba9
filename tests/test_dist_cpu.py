"""Multi-process (gloo, world size 2) coverage of the source-partitioned path, on CPU.

The GPU kernels are not available here, so each rank's partial bc comes from the oracle on
that rank's slice; what is tested is the product's host logic (paper_conf_icppw_artiless21_b200
.dist.partition / shard_sum): every source lands on exactly one rank and the all-reduce of the
partials equals the single-process result (Eq. 3: bc is a sum over sources).
"""
import os
import socket

import numpy as np
import pytest

from paper_conf_icppw_artiless21_b200 import dist as tdist


@pytest.mark.parametrize("k", [0, 1, 2, 7, 1024, 4097])
@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_partition_covers_each_source_once(k, world):
    seen = []
    for r in range(world):
        lo, hi = tdist.partition(k, world, r)
        assert 0 <= lo <= hi <= k
        assert hi - lo in (k // world, (k + world - 1) // world)
        seen.extend(range(lo, hi))
    assert seen == list(range(k))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    import torch
    import torch.distributed as dist
    import graphgen as gg
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = gg.kronecker(9, 8, seed=21, directed=True)
    src = gg.sources(g, 37, seed=3)

    def partial(s):
        return torch.from_numpy(oracle.bc(g.col_ptr, g.row_idx, True, s, nthreads=1))

    red = tdist.shard_sum(src, partial)
    np.save(os.path.join(out_dir, f"bc_{rank}.npy"), red.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_shard_sum_equals_single_process(tmp_path):
    import torch.multiprocessing as mp
    import graphgen as gg
    import oracle
    port = _free_port()
    mp.spawn(_worker, args=(2, port, str(tmp_path)), nprocs=2, join=True)
    g = gg.kronecker(9, 8, seed=21, directed=True)
    src = gg.sources(g, 37, seed=3)
    want = oracle.bc(g.col_ptr, g.row_idx, True, src, nthreads=1)
    for r in range(2):
        got = np.load(tmp_path / f"bc_{r}.npy")
        np.testing.assert_allclose(got, want, rtol=1e-12, atol=1e-12)
