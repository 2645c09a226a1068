#!/bin/bash
# ncu evidence for the current default path (run under gpurun): launch list of 2 bench steps and
# one full capture of the DELETEMIN (bgpq_dtop_kernel) launch of a C2 step.
cd "$GRAFT_REPO_ROOT"
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dtop.csv \
  python bench.py --profile-steps 2 > gpurun_out/ncu_launch.log 2>&1; echo "launch list rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bgpq_dtop -c 1 \
  -o gpurun_out/prof_dtop -f python bench.py --profile-steps 1 > gpurun_out/ncu_full.log 2>&1; echo "full rc=$?"
ls -la gpurun_out/
