#!/bin/bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
for mb in 4 8 16 32 64; do
  MCL_BATCH_MIN_BLOCKS=$mb timeout 300 python bench.py --workload cfg2 --steps 10 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('minblocks', $mb, 'threads', d['config']['threads'], 'ms', round(d['ms_per_step'],4), 'frac', round(d['roofline']['frac'],3), 'kernel_ms', round(d['roofline']['kernel_ms'],4))"
done
