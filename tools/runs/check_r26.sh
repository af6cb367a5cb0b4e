mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=10000
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k flag_rings > gpurun_out/r26_tests.txt 2>&1
bash tools/repro_synth.sh
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all.txt 2>&1
python bench.py > gpurun_out/bench_r26.json 2> gpurun_out/bench_r26.err
