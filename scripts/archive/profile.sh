#!/bin/bash
# ncu evidence for the dominant kernels (one GPU). Usage: scripts/profile.sh [workloads...]
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
for wl in ${@:-cfg5}; do
  # launch list of the bench command itself (cold-cache, serialised: compare shares)
  timeout 600 $NCU --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches_$wl.csv python bench.py --workload $wl --steps 2 --warmup 3 --no-cpu-baseline \
      > gpurun_out/launches_$wl.log 2>&1
  # one full capture of the search kernel
  timeout 900 $NCU --set full --clock-control none --import-source on -k regex:search_ -s 2 -c 1 \
      -o gpurun_out/prof_$wl -f python scripts/profile_run.py $wl 3 > gpurun_out/prof_$wl.log 2>&1
  echo "$wl done rc=$?"
done
