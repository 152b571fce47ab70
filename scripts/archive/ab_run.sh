#!/bin/bash
# A/B kernel timing of ab/libmcl_head.so (a reference build) against the in-tree build,
# after the GPU test suite; outputs in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.txt
tail -3 gpurun_out/pytest_gpu.txt
python scripts/ab_kernel.py --libs ab/libmcl_head.so paper_conf_cluster_ajipbf15_b200/libmcl.so \
    --workloads ${AB_WORKLOADS:-cfg5 cfg4 cfg2} --rounds ${AB_ROUNDS:-4} > gpurun_out/ab.txt 2>&1
cat gpurun_out/ab.txt
