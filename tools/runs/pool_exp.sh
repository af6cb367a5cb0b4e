mkdir -p gpurun_out
export RESCCL_TIMEOUT_MS=20000
rm -f gpurun_out/pool_exp.txt
for o in "instances=37 nwarps=8 tmastages=2 tmatile=12288" "instances=36 nwarps=8 tmastages=2 tmatile=14336" "instances=37 nwarps=8 tmastages=2 tmatile=14336" "instances=36 nwarps=8 tmastages=2 tmatile=12288 chunkbytes=33554432" "instances=36 nwarps=8 tmastages=2 tmatile=12288 chunkbytes=8388608" "instances=18 nwarps=16 tmastages=4 tmatile=12288 poolcap=6"; do
  echo "== $o" >> gpurun_out/pool_exp.txt
  PHASE_OPTS="chunkbytes=16777216 fifodepth=2 direct=1 $o" timeout 300 python tools/phases.py 2>&1 | head -3 >> gpurun_out/pool_exp.txt
done
