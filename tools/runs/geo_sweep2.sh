# lane engine: bigger tiles / deeper pools at one CTA per SM
mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/geo_sweep2.jsonl
: > $O
SMB_INST=1,4,8,12,16,18 timeout 900 python tools/sm_budget.py 256 w8s4t12288 w8s2t24576 w16s2t24576 w8s3t16384 w4s4t12288 w8s6t8192 >> $O 2>&1
for c in reducescatter allgather; do
SMB_COLL=$c SMB_INST=1,4,18 timeout 300 python tools/sm_budget.py 256 w8s4t12288 w8s2t24576 >> $O 2>&1
done
cat $O
