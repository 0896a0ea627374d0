"""The N>1 host path on CPU: two gloo ranks shard a scene with the C-ABI
shard ranges, each computes its slice (here with the oracle -- the device
kernel is covered by the GPU tests), and the break-map gather plus the
max-over-ranks timing reduce reassemble exactly the single-process result."""
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


def _worker(rank, world, port, P, result_dir):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_icde_giesekerhvo20_b200 import parallel, synth
    spec = synth.StackSpec(P=P, N=60, n_hist=30, k=1, miss=0.3, seed=9)
    Y, dates = synth.generate(spec, "cpu")
    b, e = parallel.shard(P, rank, world)
    out = oracle.monitor(np.ascontiguousarray(Y.numpy()[:, b:e]), dates, 30, 1, 0.25, 1.65)
    lb = torch.tensor(out["break"])
    lm = torch.tensor(out["magnitude"], dtype=torch.float32)
    gb, gm = parallel.gather_break_map(lb, lm, P)
    tmax = parallel.max_over_ranks(float(rank + 1) * 1.5)
    if rank == 0:
        np.save(os.path.join(result_dir, "gb.npy"), gb.numpy())
        np.save(os.path.join(result_dir, "gm.npy"), gm.numpy())
        np.save(os.path.join(result_dir, "tmax.npy"), np.array([tmax]))
    dist.destroy_process_group()


@pytest.mark.parametrize("P", [1000, 300])
def test_two_rank_shard_and_gather(tmp_path, P):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), P, str(tmp_path)), nprocs=world, join=True)
    import oracle
    from paper_conf_icde_giesekerhvo20_b200 import synth
    spec = synth.StackSpec(P=P, N=60, n_hist=30, k=1, miss=0.3, seed=9)
    Y, dates = synth.generate(spec, "cpu")
    ref = oracle.monitor(Y.numpy(), dates, 30, 1, 0.25, 1.65)
    gb = np.load(tmp_path / "gb.npy")
    gm = np.load(tmp_path / "gm.npy")
    assert gb.shape == (P,)
    np.testing.assert_array_equal(gb, ref["break"])
    np.testing.assert_array_equal(gm, ref["magnitude"].astype(np.float32))
    assert float(np.load(tmp_path / "tmax.npy")[0]) == 3.0


def test_sharded_generation_reassembles_the_scene():
    """Strong scaling (configs[3]): each rank generates only its shard; the
    shards equal the single-process scene column for column."""
    import torch
    from paper_conf_icde_giesekerhvo20_b200 import binding, synth
    for mask in ("iid", "cloud"):
        spec = synth.StackSpec(P=2 * synth.BLOCK + 1000, N=12, n_hist=6, miss=0.5, mask=mask, seed=13)
        full, _ = synth.generate(spec, "cpu")
        for world in (2, 3):
            parts = []
            for r in range(world):
                b, e = binding.shard_range(spec.P, r, world)
                Ys, _ = synth.generate(spec, "cpu", columns=(b, e))
                parts.append(Ys)
            got = torch.cat(parts, dim=1)
            assert torch.equal(torch.nan_to_num(got, 7.0), torch.nan_to_num(full, 7.0)), (mask, world)
