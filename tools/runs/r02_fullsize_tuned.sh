mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=30000
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -k "hm" > gpurun_out/pytest_fullsize_tuned.log 2>&1; echo "pytest=$?" >> gpurun_out/pytest_fullsize_tuned.log
tail -n 3 gpurun_out/pytest_fullsize_tuned.log
