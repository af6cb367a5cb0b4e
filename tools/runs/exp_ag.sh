mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/exp_ag.jsonl
: > $O
G="nwarps=16 tmastages=4 tmatile=12288 chunkbytes=33554432 fifodepth=2 direct=1"
for c in allgather reducescatter allreduce; do
  for ip in 0 1; do timeout 60 python tools/exp_ag.py $c 8 256 $ip "instances=4 $G" >> $O 2>&1; done
  timeout 60 python tools/exp_ag.py $c 8 256 0 "instances=4 $G storelag=4" >> $O 2>&1
  timeout 60 python tools/exp_ag.py $c 8 256 0 "instances=4 $G storelag=2" >> $O 2>&1
  timeout 60 python tools/exp_ag.py $c 2 256 0 "instances=16 $G" >> $O 2>&1
  timeout 60 python tools/exp_ag.py $c 8 256 0 "instances=4 $G" trace >> $O 2>&1
done
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/parity7.log 2>&1; tail -2 gpurun_out/parity7.log
cat $O
