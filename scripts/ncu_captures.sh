#!/bin/bash
# ncu --set full captures (source-correlated) of the dominant kernels, one GPU:
#   scripts/ncu_captures.sh [cfg5 cfg4 cfg2 cfg3 costs]   -> gpurun_out/prof_<wl>.ncu-rep
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
# launch list of the default bench command (every config): cold-cache, serialised per launch
MCL_BENCH_NO_RESIDENT=1 timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_default.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline \
    > gpurun_out/launches_default.log 2>&1
echo "launch list rc=$?"
for wl in ${@:-cfg5 cfg4 cfg2 cfg3 costs cfg5c}; do
  if [ "$wl" = costs ]; then
    timeout 900 $NCU --set full --clock-control none --import-source on -k regex:build_costs -s 2 -c 1 \
        -o gpurun_out/prof_costs -f python scripts/profile_costs.py > gpurun_out/prof_costs.log 2>&1
  else
    timeout 900 $NCU --set full --clock-control none --import-source on -k regex:search_ -s 2 -c 1 \
        -o gpurun_out/prof_$wl -f python scripts/profile_run.py $wl 3 > gpurun_out/prof_$wl.log 2>&1
  fi
  echo "$wl rc=$?"
done
