#!/bin/bash
# ncu source-level capture of one DELETEMIN cluster-engine launch (2^24 keys, K = 1024)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
timeout 300 python tools/ds_timers.py 24 1024 > gpurun_out/ds_plain.log 2>&1 || exit 1
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:bgpq_dsys_kernel -c 1 \
  -o gpurun_out/ncu_dsrc python tools/ds_timers.py 24 1024 > gpurun_out/ncu_dsrc.log 2>&1
echo "capture rc=$?"
$NCU -i gpurun_out/ncu_dsrc.ncu-rep --page source --csv --print-source sass > gpurun_out/dsrc_sass.csv 2>/dev/null
$NCU -i gpurun_out/ncu_dsrc.ncu-rep --page source --csv > gpurun_out/dsrc_cuda.csv 2>/dev/null
ls -la gpurun_out/dsrc_*; rm -f gpurun_out/ncu_dsrc.ncu-rep
