#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on small runs of every kernel path.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
run() {  # tool, workload, reps, [epochs]
  timeout 900 $CS --tool $1 --error-exitcode 9 python scripts/profile_run.py $2 $3 $4 > gpurun_out/sanitize_$1_$2_$4.log 2>&1
  echo "$1 $2 rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/sanitize_$1_$2_$4.log | tail -1)"
}
for tool in memcheck racecheck synccheck; do
  run $tool cfg1 1
  run $tool cfg2 1 64
  run $tool cfg3 1 5000
done
run memcheck cfg4 1
# warp-per-epoch batched kernel: one whole wave (2368 warps) plus split tail epochs
run memcheck cfg2 1 2400
run racecheck cfg2 1 2400
run synccheck cfg2 1 2400
# pipelined staging of host-resident batches (copies / searches / copies on three streams)
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_pipeline_gpu.py -m gpu -q -p no:cacheprovider > gpurun_out/sanitize_memcheck_pipeline.log 2>&1
echo "memcheck pipeline rc=$? $(grep -E 'ERROR SUMMARY' gpurun_out/sanitize_memcheck_pipeline.log | tail -1) $(grep -E 'passed|failed' gpurun_out/sanitize_memcheck_pipeline.log | tail -1)"
timeout 900 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_pipeline_gpu.py -m gpu -q -p no:cacheprovider -k "share_scratch or chunks_cfg2" > gpurun_out/sanitize_racecheck_pipeline.log 2>&1
echo "racecheck pipeline rc=$? $(grep -E 'RACECHECK SUMMARY' gpurun_out/sanitize_racecheck_pipeline.log | tail -1) $(grep -E 'passed|failed' gpurun_out/sanitize_racecheck_pipeline.log | tail -1)"
# round-2 paths: mixed-radix constrained kernel, packed-key merge, static policy, sockets,
# zero-copy small calls
for tool in memcheck racecheck synccheck; do
  timeout 1200 $CS --tool $tool --error-exitcode 9 python scripts/sanitize_cases.py > gpurun_out/sanitize_${tool}_r02.log 2>&1
  echo "$tool r02 cases rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/sanitize_${tool}_r02.log | tail -1)"
done
# resident mapper (one warp polling a pinned host mailbox; tagged result records)
timeout 600 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_resident_gpu.py -m gpu -q -p no:cacheprovider -k "errors or 4-3 or back_to_back" > gpurun_out/sanitize_memcheck_resident.log 2>&1
echo "memcheck resident rc=$? $(grep -E 'ERROR SUMMARY' gpurun_out/sanitize_memcheck_resident.log | tail -1) $(grep -E 'passed|failed' gpurun_out/sanitize_memcheck_resident.log | tail -1)"
timeout 600 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_resident_gpu.py -m gpu -q -p no:cacheprovider -k "4-3" > gpurun_out/sanitize_racecheck_resident.log 2>&1
echo "racecheck resident rc=$? $(grep -E 'RACECHECK SUMMARY' gpurun_out/sanitize_racecheck_resident.log | tail -1) $(grep -E 'passed|failed' gpurun_out/sanitize_racecheck_resident.log | tail -1)"
