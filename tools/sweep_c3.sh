#!/bin/bash
# Config C3 (BASELINE.json configs[2]) and the NEXT-3 K extension: 2^26 keys x {uniform,
# ascending, descending, gaussian} x K in {128 .. 4096}, keys only (under gpurun)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
: > gpurun_out/sweep_c3.jsonl
for d in uniform ascending descending gaussian; do
  for k in 128 256 512 1024 2048 4096; do
    timeout 300 python bench.py --n-log2 26 --K $k --dist $d --steps 3 --warmup 2 --no-cpu-baseline --no-e2e --no-mix 2>/dev/null | tail -1 >> gpurun_out/sweep_c3.jsonl
  done
done
wc -l gpurun_out/sweep_c3.jsonl
