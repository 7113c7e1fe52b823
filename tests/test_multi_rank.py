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


def test_shard_strong():
    """Config 5 (global batch 64, strong scaling): contiguous blocks covering every image once."""
    for world in (1, 2, 3, 4, 8):
        parts = [sharding.shard_strong(r, world, 64) for r in range(world)]
        assert sum(parts, []) == list(range(64))
        assert max(map(len, parts)) - min(map(len, parts)) <= 1
    assert sharding.shard_strong(1, 8, 64) == list(range(8, 16))
    with pytest.raises(ValueError):
        sharding.shard_strong(0, 8, 4)


def _stack_worker(rank, world, port, out_dir):
    """Two-layer stack (stride-2 then stride-1, each fed by its offset branch) on a strong shard
    of a global batch of 4 images; rank 0 gathers the last layer's y."""
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    oracle.set_num_threads(1)
    imgs = sharding.shard_strong(rank, world, 4)
    ys = []
    for c in _tiny_stack(len(imgs)):
        x = inputs.gen_x(c, imgs)
        P = inputs.gen_offset_branch(c)
        off, msk = oracle.offset_branch(x, P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"], P["pw_b"],
                                        K=c.K, G=c.G, with_mask=True, stride=c.stride, pad=c.pad)
        w, b = inputs.gen_weight(c)
        ys.append(oracle.dcn_forward(x, off, w, b, mask=msk, stride=c.stride, pad=c.pad))
    t = torch.from_numpy(np.ascontiguousarray(ys[-1]))
    yall = sharding.gather_outputs(dist, t)
    if rank == 0:
        np.save(os.path.join(out_dir, "stack.npy"), yall.numpy())
    dist.barrier()
    dist.destroy_process_group()


def _tiny_stack(n):
    return [configs.LayerConfig("ts0", N=n, Cin=8, Cout=8, H=9, W=7, stride=2, config_id=12),
            configs.LayerConfig("ts1", N=n, Cin=8, Cout=8, H=5, W=4, config_id=12)]


def test_gloo_strong_sharding_stack(tmp_path, oracle_mod):
    world = 2
    mp.spawn(_stack_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    c = _tiny_stack(4)[-1]
    x = inputs.gen_x(c)
    P = inputs.gen_offset_branch(c)
    off, msk = oracle_mod.offset_branch(x, P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"], P["pw_b"],
                                        K=c.K, G=c.G, with_mask=True, stride=c.stride, pad=c.pad)
    w, b = inputs.gen_weight(c)
    ref = oracle_mod.dcn_forward(x, off, w, b, mask=msk, stride=c.stride, pad=c.pad)
    assert np.array_equal(np.load(tmp_path / "stack.npy"), ref)
