#!/bin/bash
# C2 50/50 concurrent mix (paper E4 shape) evidence (run under gpurun)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 300 python bench.py --mix --n-log2 20 --prefill-log2 16 --steps 3 --warmup 3 > gpurun_out/mix_small.log 2>&1; echo "mix small rc=$?"; tail -c 600 gpurun_out/mix_small.log
timeout 900 python bench.py --mix --steps 3 --warmup 3 > gpurun_out/mix_w4.log 2>&1; echo "mix w4 rc=$?"
timeout 900 python bench.py --mix --values --steps 3 --warmup 3 > gpurun_out/mix_w8.log 2>&1; echo "mix w8 rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_mix.csv python bench.py --mix --steps 1 --warmup 3 > /dev/null 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bgpq_locks -c 1 -o gpurun_out/prof_mix -f python bench.py --mix --n-log2 24 --prefill-log2 20 --steps 1 --warmup 3 > gpurun_out/ncu_mix.log 2>&1; echo "ncu full mix rc=$?"
