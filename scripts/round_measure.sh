#!/bin/bash
# Round measurements on one GPU (outputs in gpurun_out/):
#   bench.json           default bench line (cfg5 headline + configs{cfg1..cfg4}, CPU oracle)
#   bench_2ranks.json    2 ranks sharing the one GPU (gloo control plane, fused exchange)
#   bench_2ranks_nccl.*  the same with --collective nccl (may be refused on one GPU)
#   bench_4ranks.json    4 ranks sharing the one GPU (fused exchange at world 4)
#   resident_latency.jsonl  cfg1 decision latency: resident warp vs a launch per call
#   scaling.jsonl        projected strong scaling from per-rank shard kernels
#   variants.jsonl       NEXT-1..4 variants (constrained, policies, pruned, cost tables)
#   costs.jsonl          cost-table kernel, L2 flushed
#   fuzz_parity.json     randomised GPU-vs-oracle sweep (120 s)
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29541 bench.py --gpus 2 --collective fused --steps 5 --warmup 3 \
    > gpurun_out/bench_2ranks.json 2> gpurun_out/bench_2ranks.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29542 bench.py --gpus 2 --collective nccl --only --workload cfg4 --steps 5 --warmup 3 \
    > gpurun_out/bench_2ranks_nccl.json 2> gpurun_out/bench_2ranks_nccl.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 \
    --master-port 29543 bench.py --gpus 4 --collective fused --steps 5 --warmup 3 --no-cpu-baseline \
    > gpurun_out/bench_4ranks.json 2> gpurun_out/bench_4ranks.err
timeout 300 python scripts/resident_latency.py > gpurun_out/resident_latency.jsonl 2>&1
timeout 600 python scripts/scaling_model.py > gpurun_out/scaling.jsonl 2>&1
timeout 900 python scripts/bench_variants.py --reps 7 > gpurun_out/variants.jsonl 2>&1
timeout 300 python scripts/bench_costs.py > gpurun_out/costs.jsonl 2>&1
timeout 300 python scripts/fuzz_parity.py 120 $RANDOM > gpurun_out/fuzz_parity.json 2>&1
echo done
