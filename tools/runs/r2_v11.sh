mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 2400 python -m pytest tests/test_gpu_robustness.py tests/test_gpu_api_rules.py tests/test_gpu_fullsize.py tests/test_gpu_parity_r2.py -m gpu -q > gpurun_out/r2v11_pytest.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v11_pytest.log
tail -5 gpurun_out/r2v11_pytest.log
