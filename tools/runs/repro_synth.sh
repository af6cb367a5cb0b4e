mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=5000
{
python tools/repro.py synth reducescatter 8 524288 "seed=0 fanout=2" \
 "chunkbytes=1048576 fifodepth=2 instances=4 direct=1" ";" \
 "chunkbytes=1048576 fifodepth=2 instances=4 direct=1 tma=0" ";" \
 "chunkbytes=1048576 fifodepth=2 instances=4 direct=1 tmamin=100000000" ";" \
 "chunkbytes=4194304 fifodepth=2 instances=4 direct=1" ";" \
 "chunkbytes=1048576 fifodepth=2 instances=4 direct=0" ";" \
 "chunkbytes=1048576 fifodepth=2 instances=1 direct=1" ";" \
 "chunkbytes=262144 fifodepth=2 instances=1 direct=1 tma=0"
} > gpurun_out/repro_synth.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_multiprocess.py -q -x -k windows > gpurun_out/windows.txt 2>&1
