#!/bin/bash
# ncu evidence of the round-2 build (under gpurun, one GPU): launch list of the bench command,
# --set full captures of the DELETEMIN cluster kernel and the INSERT pipeline kernel at C2
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches_r2.csv python bench.py --profile-steps 2 > gpurun_out/launches_r2.log 2>&1
echo "launch list rc=$?"
timeout 1500 $NCU --set full --clock-control none --import-source on -k regex:bgpq_dsys_kernel -s 1 -c 1 \
  -o gpurun_out/ncu_dsys python bench.py --profile-steps 2 > gpurun_out/ncu_dsys.log 2>&1
echo "dsys capture rc=$?"
timeout 1500 $NCU --set full --clock-control none --import-source on -k regex:bgpq_ins_pipe2_kernel -s 1 -c 1 \
  -o gpurun_out/ncu_pipe2 python bench.py --profile-steps 2 > gpurun_out/ncu_pipe2.log 2>&1
echo "pipe2 capture rc=$?"
for r in ncu_dsys ncu_pipe2; do
  [ -f gpurun_out/$r.ncu-rep ] && python tools/ncu_summary.py gpurun_out/$r.ncu-rep gpurun_out/$r.summary.json > /dev/null
  [ -f gpurun_out/$r.ncu-rep ] && $NCU -i gpurun_out/$r.ncu-rep --page source --csv > gpurun_out/$r.source.csv 2>/dev/null
done
bash tools/ncu_export.sh
