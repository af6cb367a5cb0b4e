mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=300000
CS=/usr/local/cuda/bin/compute-sanitizer
for t in memcheck synccheck racecheck; do
  echo "== $t" >> gpurun_out/san_tma.txt
  SMALL_RUN_TMA=1 timeout 1200 $CS --tool $t --error-exitcode 3 python tools/small_run.py > gpurun_out/san_tma_$t.log 2>&1
  echo "rc=$?" >> gpurun_out/san_tma.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|ALL OK|FAILED" gpurun_out/san_tma_$t.log | tail -3 >> gpurun_out/san_tma.txt
done
