mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
bash tools/exp_tr2.sh
O=gpurun_out/exp_fix1.jsonl
: > $O
for o in "tmastages=4 tmatile=12288" "tmastages=2 tmatile=24576" "tmastages=4 tmatile=8192" "tmastages=8 tmatile=6144"; do
  for c in reducescatter allgather allreduce; do
    SMB_COLL=$c SMB_INST=4 SMB_OPTS="$o" timeout 120 python tools/sm_budget.py 256 one >> $O 2>&1
  done
done
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/parity_fix1.log 2>&1; tail -2 gpurun_out/parity_fix1.log
