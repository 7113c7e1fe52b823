"""Multi-process (gloo, world size 2, CPU) tests of the data-parallel sharding logic.

The GPU path shards images across ranks with no data-path collective.
Here each rank regenerates its shard from the per-image seeds and runs the fp64 oracle on it;
rank 0 gathers the per-image outputs and checks they equal a single-process run, and the
max-over-ranks time reduction is checked.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from defcon_workloads import configs, inputs, sharding


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    oracle.set_num_threads(1)
    c = configs.LayerConfig("mr", N=2, Cin=8, Cout=8, H=6, W=5, config_id=11)
    imgs = sharding.shard_images(rank, world, c.N)
    x = inputs.gen_x(c, imgs)
    off = inputs.gen_offsets(c, imgs)
    msk = inputs.gen_mask(c, imgs)
    w, b = inputs.gen_weight(c)
    y = oracle.dcn_forward(x, off, w, b, mask=msk)
    t = torch.from_numpy(np.ascontiguousarray(y))
    gathered = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(gathered, t)
    mx = sharding.max_over_ranks(dist, [float(rank + 1), 10.0 - rank], "cpu")
    cks = sharding.gather_checksums(dist, sharding.image_checksums(t))
    yall = sharding.gather_outputs(dist, t)
    if rank == 0:
        np.save(os.path.join(out_dir, "sharded.npy"), torch.cat(gathered).numpy())
        np.save(os.path.join(out_dir, "max.npy"), np.array(mx))
        np.save(os.path.join(out_dir, "cks.npy"), cks.numpy())
        np.save(os.path.join(out_dir, "yall.npy"), yall.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_sharding_matches_single_process(tmp_path, oracle_mod):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    sharded = np.load(tmp_path / "sharded.npy")
    c = configs.LayerConfig("mr", N=2 * world, Cin=8, Cout=8, H=6, W=5, config_id=11)
    L = inputs.gen_layer(c)
    ref = oracle_mod.dcn_forward(L["x"], L["offset"], L["weight"], L["bias"], mask=L["mask"])
    assert np.array_equal(sharded, ref)          # bitwise: same images, same order
    assert list(np.load(tmp_path / "max.npy")) == [2.0, 10.0]
    # the gathered per-image checksums equal those of the single-process result (invariance),
    # and the output gather reproduces it
    single = sharding.image_checksums(torch.from_numpy(np.ascontiguousarray(ref))).numpy()
    assert np.array_equal(np.load(tmp_path / "cks.npy"), single)
    assert np.array_equal(np.load(tmp_path / "yall.npy"), ref)


def test_shard_images():
    assert sharding.shard_images(1, 4, 16) == list(range(16, 32))
    with pytest.raises(ValueError):
        sharding.shard_images(4, 4, 16)
