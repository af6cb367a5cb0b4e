mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
G="nwarps=16 tmastages=4 tmatile=12288 chunkbytes=33554432 fifodepth=2 direct=1 trace=2 ring=1"
timeout 120 python tools/exp_ag.py reducescatter 8 256 0 "instances=4 $G" > gpurun_out/tr2_rs.txt 2>&1
timeout 120 python tools/exp_ag.py allgather 8 256 0 "instances=4 $G" > gpurun_out/tr2_ag.txt 2>&1
tail -3 gpurun_out/tr2_rs.txt; tail -3 gpurun_out/tr2_ag.txt
O=gpurun_out/exp_ring.jsonl
: > $O
for o in "ring=1 tmastages=4 tmatile=12288" "ring=1 tmastages=4 tmatile=24576" "ring=1 tmastages=2 tmatile=24576" "ring=1 tmastages=3 tmatile=16384" "ring=1 tmastages=8 tmatile=6144"; do
  for c in reducescatter allgather allreduce; do
    SMB_COLL=$c SMB_INST=4 SMB_OPTS="$o" timeout 120 python tools/sm_budget.py 256 one >> $O 2>&1
  done
done
RESCCL_RING=1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/parity_ring.log 2>&1; tail -2 gpurun_out/parity_ring.log
