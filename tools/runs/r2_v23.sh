mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2v23_smoke.log 2>&1
timeout 2700 python -m pytest tests -m gpu -q > gpurun_out/r2v23_pytest_all.log 2>&1; echo "pytest=$?" >> gpurun_out/r2v23_pytest_all.log
tail -6 gpurun_out/r2v23_pytest_all.log; tail -1 gpurun_out/r2v23_smoke.log
