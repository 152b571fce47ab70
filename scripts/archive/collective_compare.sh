#!/bin/bash
# Per-step cost of the cross-GPU combine on one GPU: no collective vs a 1-rank NCCL
# all-reduce + decode kernel vs the fused in-kernel peer exchange (NEXT-2).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
out=gpurun_out/collective_compare.jsonl
: > $out
for wl in ${WORKLOADS:-cfg1 cfg4 cfg5}; do
  for c in auto nccl fused; do
    timeout 300 python bench.py --workload $wl --collective $c --steps 20 --warmup 5 --no-cpu-baseline \
      2> gpurun_out/cc_${wl}_${c}.err | tail -1 >> $out
  done
done
python - <<'PY'
import json
for l in open("gpurun_out/collective_compare.jsonl"):
    d = json.loads(l)
    c = d["config"]
    print(f'{c["workload"]:5s} {c.get("combine","?"):6s} ms/step {d["ms_per_step"]:.4f} kernel_ms {d["roofline"]["kernel_ms"]:.4f} '
          f'launches/step {d["gpu_launches"]/d["steps"]:.0f} e2e_ms {d["e2e"]["ms_per_step"]:.4f}')
PY
