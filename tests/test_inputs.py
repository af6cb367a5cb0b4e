"""The shared input recipe: the torch (device) evaluation is bit-identical to numpy."""
import numpy as np
import pytest

import resccl_inputs as inp


@pytest.mark.parametrize("dtype", ["int32", "float32", "float16", "bfloat16"])
@pytest.mark.parametrize("mode", ["uniform", "exact"])
def test_torch_generator_matches_numpy(dtype, mode):
    import torch
    for rank in (0, 5):
        a = inp.rank_input(dtype, 7, rank, 5000, mode)
        t = inp.rank_input_torch(dtype, 7, rank, 5000, device="cpu", mode=mode, block=1234)
        b = t.view(torch.int16).numpy().view(np.uint16) if dtype == "bfloat16" else t.numpy()
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8))
        idx = np.array([0, 17, 4999, 123])
        c = inp.rank_input_at(dtype, 7, rank, idx, mode)
        assert np.array_equal(c.view(np.uint8), a[idx].view(np.uint8))
