"""Multi-process batch sharding on CPU (world_size 2, gloo).

Each rank runs its contiguous shard of the global batch -- here through the
oracle, since the CPU box has no GPU -- and the logits are all-gathered with
the same helper bench.py uses on NCCL.  The gathered logits must equal the
single-process run of the whole batch bit for bit (images are independent;
the GPU kernels are batch-invariant too, see test_gpu_parity)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_songljkj0024_b200.shard import gather_logits, shard_range


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, per_rank, out_path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import workloads as W
    m = W.resnet18_cifar(batch=per_rank, dtype="f32", height=16, width=16)
    start, stop = shard_range(rank, world, per_rank)
    x = W.make_input(m, start=start, count=stop - start)
    local = torch.from_numpy(oracle.run_temco(oracle.plan(m), x).astype(np.float32))
    full = gather_logits(local, world)
    if rank == 0:
        np.save(out_path, full.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_shard_range():
    assert shard_range(0, 4, 256) == (0, 256)
    assert shard_range(3, 4, 256) == (768, 1024)
    with pytest.raises(ValueError):
        shard_range(4, 4, 256)


def test_two_rank_gather_equals_single_process(tmp_path):
    import oracle
    import workloads as W
    world, per_rank = 2, 3
    out = str(tmp_path / "gathered.npy")
    mp.spawn(_worker, args=(world, _free_port(), per_rank, out), nprocs=world, join=True)
    got = np.load(out)
    m = W.resnet18_cifar(batch=world * per_rank, dtype="f32", height=16, width=16)
    ref = oracle.run_temco(oracle.plan(m), W.make_input(m)).astype(np.float32)
    assert got.shape == ref.shape
    np.testing.assert_allclose(got, ref, rtol=1e-6, atol=1e-7)   # BLAS blocking may differ by batch
