# r02: C2 (ring AR/AG 1 KiB - 1 GiB), C4 (synth AG/RS), and ring AR at 2/4/8 virtual ranks on the device clock
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=60000
timeout 2400 python tools/sweep.py c2 > gpurun_out/r2v28_c2.jsonl 2> gpurun_out/r2v28.err
timeout 1200 python tools/sweep.py nr > gpurun_out/r2v28_nr.jsonl 2>> gpurun_out/r2v28.err
timeout 1200 python tools/sweep.py c4 > gpurun_out/r2v28_c4.jsonl 2>> gpurun_out/r2v28.err
wc -l gpurun_out/r2v28_*.jsonl; tail -3 gpurun_out/r2v28.err
