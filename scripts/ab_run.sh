cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python scripts/ab_kernel.py --libs ab/libmcl_head.so paper_conf_cluster_ajipbf15_b200/libmcl.so --workloads cfg5 cfg4 cfg2 --rounds 4 > gpurun_out/ab1.txt 2>&1
for wl in cfg4 cfg2; do
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:search_ -s 2 -c 1 -o gpurun_out/prof_new_$wl -f python scripts/profile_run.py $wl 3 > /dev/null 2>&1
done
cat gpurun_out/ab1.txt
