#!/bin/bash
# Evidence of the late round-2 build (under gpurun, one GPU): bench line, ncu launch lists of the
# bench and of one C2 mixed call, ncu --set full captures of the DELETEMIN cluster kernel, the
# INSERT pipeline kernel and the mixed call's cluster kernel; summaries + CSV exports.
cd "$GRAFT_REPO_ROOT"; mkdir -p ${OUT:-gpurun_out/late}
O=${OUT:-gpurun_out/late}
NCU=/usr/local/cuda/bin/ncu
timeout 900 python bench.py --steps 5 --warmup 3 > $O/bench.log 2>&1; echo "bench rc=$?"
timeout 600 python tools/mix_once.py > $O/mix_once.log 2>&1 || { echo "mix_once failed"; exit 1; }
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file $O/launches.csv python bench.py --profile-steps 2 > $O/launches.log 2>&1; echo "launch list rc=$?"
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file $O/launches_mix.csv python tools/mix_once.py > $O/launches_mix.log 2>&1; echo "mix launch list rc=$?"
for spec in "dsys:bgpq_dsys_kernel:bench.py --profile-steps 2" "pipe2:bgpq_ins_pipe2_kernel:bench.py --profile-steps 2" "mixdsys:bgpq_dsys_kernel:tools/mix_once.py"; do
  IFS=: read name kern cmd <<< "$spec"
  timeout 1500 $NCU --set full --clock-control none --import-source on -k regex:$kern -s 1 -c 1 \
    -o $O/ncu_$name python $cmd > $O/ncu_$name.log 2>&1; echo "$name capture rc=$?"
  [ -f $O/ncu_$name.ncu-rep ] && python tools/ncu_summary.py $O/ncu_$name.ncu-rep $O/ncu_$name.summary.json > /dev/null
  [ -f $O/ncu_$name.ncu-rep ] && $NCU -i $O/ncu_$name.ncu-rep --page details --csv > $O/ncu_$name.details.csv 2>/dev/null
  rm -f $O/ncu_$name.ncu-rep
done
du -sh $O
