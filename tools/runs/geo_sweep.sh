# per-SM efficiency of the lane engine at low CTA counts vs stage geometry
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/geo_sweep.jsonl
: > $O
SMB_INST=1,2,4,8,18 timeout 600 python tools/sm_budget.py 256 two one w16s8t6144 w16s6t8192 w8s4t12288 w8s8t6144 w32s4t12288 >> $O 2>&1
for c in reducescatter allgather; do
SMB_COLL=$c SMB_INST=1,4 timeout 300 python tools/sm_budget.py 256 two one w16s8t6144 >> $O 2>&1
done
cat $O
