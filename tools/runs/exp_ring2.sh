mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/exp_ring2.jsonl
: > $O
SMB_INST=1,4,8,12,18 SMB_OPTS="ring=1" timeout 300 python tools/sm_budget.py 256 one two >> $O 2>&1
SMB_INST=1,4,8,12,18 SMB_OPTS="ring=1 tmastages=2 tmatile=24576" timeout 300 python tools/sm_budget.py 256 one >> $O 2>&1
SMB_INST=24,30,37 SMB_OPTS="ring=1" timeout 300 python tools/sm_budget.py 256 two >> $O 2>&1
SMB_INST=24,30,37 SMB_OPTS="ring=1 tmastages=1 tmatile=24576" timeout 300 python tools/sm_budget.py 256 two >> $O 2>&1
for b in "" "--instances 37 --nwarps 8 --chunk-bytes 33554432"; do :; done
cat $O
