mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
O=gpurun_out/exp_tile.jsonl
: > $O
for o in "tmastages=4 tmatile=12288" "tmastages=2 tmatile=24576" "tmastages=1 tmatile=49152" "tmastages=4 tmatile=8192" "tmastages=8 tmatile=6144"; do
  for c in reducescatter allgather; do
    SMB_COLL=$c SMB_INST=4 SMB_OPTS="$o" timeout 120 python tools/sm_budget.py 256 one >> $O 2>&1
  done
done
cat $O
