"""The sharded path's NCCL leg on one GPU:
a 1-process torch.distributed group bootstraps the library's own NCCL
communicator (ShardComm: rank 0's ncclGetUniqueId broadcast through the
process group), and plr_execute_sharded runs its ncclAllGather of the 64-byte
payload over that 1-rank communicator.  The concatenation-equals-oracle
reading R12 is checked element by element, and the result equals the
communicator-less loopback of the same schedule."""
import os
import socket

import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module")
def group():
    import torch
    import torch.distributed as dist
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")     # one rank: the bootstrap stays on loopback
    dist.init_process_group("nccl", init_method="tcp://127.0.0.1:%d" % _free_port(), rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    yield dist
    dist.destroy_process_group()


@pytest.mark.parametrize("name", ["prefix", "order3", "tuple2", "hp3", "lp2"])
@pytest.mark.parametrize("n", [40 * 3840 + 17, (1 << 23) + 5])
def test_sharded_nccl_world1(cuda_plr, group, name, n):
    import torch
    sig = workloads.BY_NAME[name]
    comm = cuda_plr.ShardComm()
    assert comm.world == 1 and comm.handle.value
    x = workloads.host_input(n, sig.dtype, 61)
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    xd = torch.from_numpy(x).cuda()
    y = plan.sharded(xd, comm=comm).cpu().numpy()

    class Loop:
        rank, world, handle = 0, 1, None
    y_loop = plan.sharded(xd, comm=Loop()).cpu().numpy()
    ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    if sig.dtype == "int32":
        assert np.array_equal(y, ref)
    else:
        assert float(np.max(np.abs(y - ref) / np.maximum(1.0, np.abs(ref)))) <= 1e-4
    assert np.array_equal(y.view(np.uint32), y_loop.view(np.uint32))
    plan.close()
    comm.close()
