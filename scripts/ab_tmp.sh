cd "${GRAFT_REPO_ROOT}"
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_batch_gpu.py -m gpu -q -x --timeout 500 -p no:cacheprovider > gpurun_out/pytest_batch.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_batch.txt
tail -2 gpurun_out/pytest_batch.txt
python scripts/ab_kernel.py --libs ab/libmcl_head.so ab/libmcl_new.so ab/libmcl_new.so@MCL_BATCH_PIECES=2 ab/libmcl_new.so@MCL_BATCH_TAIL=0 --workloads cfg2:E=2368 cfg2:E=3000 cfg2:E=4000 cfg2:E=7000 cfg2 --rounds 3 > gpurun_out/ab.txt 2>&1
cat gpurun_out/ab.txt
