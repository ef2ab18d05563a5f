cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02k
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02k/build.log 2>&1; echo build rc $?
for w in c2 c3 c4 c5; do timeout 300 python bench.py --steps 20 --warmup 5 --workload $w --no-cpu-baseline > gpurun_out/r02k/bench_$w.json 2>gpurun_out/r02k/bench_$w.err; echo bench $w rc $?; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:linear_ln_kernel -s 6 -c 1 -o gpurun_out/r02k/wo_c2 env TCB_NO_COOP=1 python bench.py --workload c2 --steps 1 --warmup 2 --no-cpu-baseline --no-graph > gpurun_out/r02k/ncu_wo.log 2>&1; echo ncu wo rc $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_tc3 -s 6 -c 1 -o gpurun_out/r02k/attn_c2 env TCB_NO_COOP=1 python bench.py --workload c2 --steps 1 --warmup 2 --no-cpu-baseline --no-graph > gpurun_out/r02k/ncu_attn.log 2>&1; echo ncu attn rc $?
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_LN_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > gpurun_out/r02k/build_probe.log 2>&1
timeout 120 python - <<'PY' 2>&1 | grep -E "lnprobe|^K" | tee gpurun_out/r02k/ln_probe.txt
import sys; sys.path.insert(0,'.')
import torch, paper_conf_icpp_fuc0z22_b200 as tcb
M,N,K=32768,512,512
A=torch.randn(M,K,device='cuda').bfloat16(); W=(torch.randn(N,K,device='cuda')*0.02).bfloat16(); b=torch.zeros(N,device='cuda')
R=torch.randn(M,N,device='cuda').bfloat16(); g=torch.ones(N,device='cuda'); be=torch.zeros(N,device='cuda')
for _ in range(2): tcb.op_linear_ln(A,W,b,R,g,be,1e-5)
torch.cuda.synchronize()
print('K',K, flush=True)
tcb.op_linear_ln(A,W,b,R,g,be,1e-5); torch.cuda.synchronize()
PY
