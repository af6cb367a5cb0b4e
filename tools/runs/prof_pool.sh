mkdir -p gpurun_out
O="instances=36 nwarps=8 tmastages=3 tmatile=8192 poolcap=3 chunkbytes=16777216 fifodepth=2 direct=1"
ncu --set full --clock-control none --import-source on -k regex:resccl -s 2 -c 1 -o gpurun_out/prof_rs_pool python tools/one_coll.py reducescatter 256 "$O" 3 > gpurun_out/prof_rs_pool.log 2>&1
ncu -i gpurun_out/prof_rs_pool.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_rs_pool_sass.csv 2>gpurun_out/prof_rs_pool_sass.err
ncu -i gpurun_out/prof_rs_pool.ncu-rep --page details --csv > gpurun_out/prof_rs_pool_details.csv 2>/dev/null
