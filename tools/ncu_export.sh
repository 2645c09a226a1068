#!/bin/bash
# Export .ncu-rep captures under gpurun_out/ to CSV (raw + source pages) and drop the
# binary reports so gpurun_out/ stays under gpurun's 64 MiB copy-back limit.
cd "$GRAFT_REPO_ROOT"
for r in gpurun_out/*.ncu-rep; do
  [ -f "$r" ] || continue
  b="${r%.ncu-rep}"
  ncu -i "$r" --page raw --csv > "$b.raw.csv" 2>/dev/null
  ncu -i "$r" --page details --csv > "$b.details.csv" 2>/dev/null
  rm -f "$r"
done
du -sh gpurun_out
