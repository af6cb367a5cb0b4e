"""f4 host logic of the torch.distributed backend (no GPU): the backend registers under
the name "resccl" for CUDA tensors and maps torch's reduce ops onto the ABI's."""
import pytest
import torch.distributed as dist


def test_backend_registered_and_op_mapping():
    import paper_conf_sigcomm_liuhlgcwz025_b200.process_group as pg
    assert "resccl" in dist.Backend.backend_list
    o = dist.AllreduceOptions()
    for op, name in ((dist.ReduceOp.SUM, "sum"), (dist.ReduceOp.MAX, "max"), (dist.ReduceOp.MIN, "min"),
                     (dist.ReduceOp.AVG, "avg")):
        o.reduceOp = op
        assert pg._op_name(o.reduceOp) == name
    o.reduceOp = dist.ReduceOp.PRODUCT
    with pytest.raises(ValueError):
        pg._op_name(o.reduceOp)
