"""Multi-GPU batch shard on NCCL: two ranks, one GPU each, each runs
its contiguous shard through its own plan on the CUDA path and the fp32 logits are
all-gathered with the NCCL all_gather_into_tensor branch of shard.gather_logits.
The gathered logits must equal a single-GPU run of the same global batch bit for
bit (images are independent; the kernels are batch-invariant).  Skipped on boxes
with fewer than two GPUs (the round-end GPU tier has one)."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, per_rank, out_path):
    import torch.distributed as dist

    import workloads as W
    from paper_conf_icpp_songljkj0024_b200 import Plan
    from paper_conf_icpp_songljkj0024_b200.shard import gather_logits, shard_range
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    m = W.resnet50(batch=per_rank, dtype="bf16", height=64, width=64)
    start, stop = shard_range(rank, world, per_rank)
    x = torch.from_numpy(W.make_input(m, start=start, count=stop - start)).cuda().to(torch.bfloat16)
    p = Plan(m)
    y = torch.empty(p.output_shape(), dtype=torch.float32, device="cuda")
    p.run(x, y)
    full = gather_logits(y, world)
    torch.cuda.synchronize()
    if rank == 0:
        np.save(out_path, full.cpu().numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2, reason="needs 2 GPUs")
def test_two_gpu_nccl_gather_equals_single_gpu(tmp_path):
    import torch.multiprocessing as mp

    import workloads as W
    from paper_conf_icpp_songljkj0024_b200 import Plan
    world, per_rank = 2, 4
    out = str(tmp_path / "gathered.npy")
    mp.spawn(_worker, args=(world, _free_port(), per_rank, out), nprocs=world, join=True)
    got = np.load(out)
    m = W.resnet50(batch=world * per_rank, dtype="bf16", height=64, width=64)
    p = Plan(m)
    x = torch.from_numpy(W.make_input(m)).cuda().to(torch.bfloat16)
    y = torch.empty(p.output_shape(), dtype=torch.float32, device="cuda")
    p.run(x, y)
    torch.cuda.synchronize()
    assert np.array_equal(got, y.cpu().numpy())
