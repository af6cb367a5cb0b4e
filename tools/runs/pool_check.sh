mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all_pool.txt 2>&1
for o in "instances=36 nwarps=8 tmastages=2 tmatile=12288" "instances=36 nwarps=8 tmastages=3 tmatile=8192" "instances=36 nwarps=8 tmastages=2 tmatile=8192" "instances=18 nwarps=16 tmastages=4 tmatile=12288" "instances=18 nwarps=16 tmastages=3 tmatile=16384"; do
  echo "== $o" >> gpurun_out/pool_exp.txt
  PHASE_OPTS="$o chunkbytes=16777216 fifodepth=2 direct=1" timeout 300 python tools/phases.py 2>&1 | head -3 >> gpurun_out/pool_exp.txt
done
