# lane engine: tiles of 24-48 KiB, 16-32 warps, one CTA per SM
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/geo_sweep3.jsonl
: > $O
SMB_INST=1,4,8,10,12,14,16,18 timeout 900 python tools/sm_budget.py 256 w16s2t24576 w32s2t24576 w16s1t49152 w32s1t49152 w16s1t32768 >> $O 2>&1
for c in reducescatter allgather; do
SMB_COLL=$c SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w16s2t24576 w32s1t49152 >> $O 2>&1
done
cat $O
