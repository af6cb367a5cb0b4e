"""f4 framework integration: ResCCL as the gradient AllReduce of PyTorch DDP.

The paper integrates ResCCL into Megatron-LM by "relink and rebuild"
and runs data-parallel gradient synchronisation through it (T5, DP = 16).
Here the equivalent hook point is DDP's communication hook: every gradient bucket is
AllReduced in place by the generated ResCCL kernels on the current stream and scaled
by 1/world; DDP keeps its own process group for everything else (parameter broadcast,
bucket rebuilding).  Argument marshalling only -- the reduction runs in libresccl.so.

    comm = init_process_group_comm(rank, world, device)
    ddp_model.register_comm_hook(ResCCLHookState(comm), resccl_allreduce_hook)
"""
import torch  # no `from __future__ import annotations`: DDP checks the hook's real annotation

from .torch_api import Communicator


class ResCCLHookState:
    def __init__(self, comm: Communicator, average: bool = True):
        self.comm = comm
        self.average = average
        self.calls = 0
        self.bytes = 0


def resccl_allreduce_hook(state: ResCCLHookState, bucket) -> torch.futures.Future[torch.Tensor]:
    """DDP comm hook: in-place ResCCL AllReduce (sum) of the flattened bucket, then / world."""
    buf = bucket.buffer()
    stream = torch.cuda.current_stream(buf.device)
    state.comm.allreduce(buf, buf, stream=stream.cuda_stream)
    if state.average:
        buf.div_(state.comm.nranks)
    state.calls += 1
    state.bytes += buf.numel() * buf.element_size()
    fut = torch.futures.Future(devices=[buf.device])
    fut.set_result(buf)
    return fut
