#!/bin/bash
# End-of-round evidence on one GPU: bench lines for every config, ncu launch lists and full
# captures of the dominant kernels, the ALU probe, sanitizer runs. Outputs in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/../..}"
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
python scripts/archive/probe_all.py > gpurun_out/probe_ops.txt 2>&1
for wl in cfg5 cfg4 cfg2 cfg3 cfg1; do
  timeout 600 python bench.py --workload $wl --only --steps 20 --warmup 5 > gpurun_out/bench_$wl.json 2> gpurun_out/bench_$wl.err
done
for wl in cfg5 cfg4 cfg2 cfg3; do
  timeout 600 $NCU --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches_$wl.csv python bench.py --workload $wl --only --steps 2 --warmup 3 --no-cpu-baseline \
      > /dev/null 2>&1
  timeout 900 $NCU --set full --clock-control none --import-source on -k regex:search_ -s 2 -c 1 \
      -o gpurun_out/prof_$wl -f python scripts/profile_run.py $wl 3 > /dev/null 2>&1
done
timeout 600 $NCU --set full --clock-control none --import-source on -k regex:build_costs -s 2 -c 1 -o gpurun_out/prof_costs -f \
    python scripts/profile_costs.py > /dev/null 2>&1
python scripts/bench_variants.py --reps 7 > gpurun_out/variants.jsonl 2>&1
python scripts/archive/pipeline_study.py > gpurun_out/pipeline_study.jsonl 2>&1
./scripts/sanitize.sh > gpurun_out/sanitize_summary.txt 2>&1
ls gpurun_out
