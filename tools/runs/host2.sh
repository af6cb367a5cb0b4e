mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 600 python -m pytest tests/test_gpu_host_buffers.py -x -q > gpurun_out/pytest_host2.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_host2.log
tail -4 gpurun_out/pytest_host2.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_v15.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_gpu_v15.log
tail -3 gpurun_out/pytest_gpu_v15.log
