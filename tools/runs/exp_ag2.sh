mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/exp_ag2.jsonl
: > $O
G="nwarps=16 tmastages=4 tmatile=12288 chunkbytes=33554432 fifodepth=2 direct=1"
for c in allgather reducescatter allreduce; do
  timeout 60 python tools/exp_ag.py $c 8 256 0 "instances=4 $G" >> $O 2>&1
  timeout 60 python tools/exp_ag.py $c 8 256 0 "instances=4 $G storelag=2" >> $O 2>&1
done
cat $O
SMB_INST=1,4,8,18 timeout 300 python tools/sm_budget.py 256 one two > gpurun_out/smb5.jsonl 2>&1
SMB_INST=24,30,37 timeout 300 python tools/sm_budget.py 256 two >> gpurun_out/smb5.jsonl 2>&1
cat gpurun_out/smb5.jsonl
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/parity8.log 2>&1; tail -2 gpurun_out/parity8.log
