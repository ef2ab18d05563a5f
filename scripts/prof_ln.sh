cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/p1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:linear_lnc_kernel -s 4 -c 2 -o gpurun_out/p1/c4_lnc python bench.py --workload c4 --steps 1 --warmup 1 --no-cpu-baseline --no-graph > gpurun_out/p1/c4.log 2>&1; echo rc $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:linear_ln -s 4 -c 2 -o gpurun_out/p1/c2_ln python bench.py --workload c2 --steps 1 --warmup 1 --no-cpu-baseline --no-graph > gpurun_out/p1/c2.log 2>&1; echo rc $?
