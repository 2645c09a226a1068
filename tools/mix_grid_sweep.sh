#!/bin/bash
# C2 mix vs persistent CTA count (paper P:416: more blocks, more lock contention)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
for g in 16 32 64 96 148; do
  timeout 400 python bench.py --mix --grid $g --steps 3 --warmup 3 > gpurun_out/mix_grid_$g.log 2>&1; echo "grid $g rc=$?"
done
