cd $GRAFT_REPO_ROOT; T=gpurun_out/probe3s; mkdir -p $T
python - <<'PY' | tee $T/d2h.txt
import torch, time
x = torch.empty(33_294_336 // 2, dtype=torch.bfloat16, device="cuda")
h = torch.empty(x.shape, dtype=torch.bfloat16).pin_memory()
for _ in range(3): h.copy_(x, non_blocking=True)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(10): h.copy_(x, non_blocking=True)
b.record(); torch.cuda.synchronize()
ms = a.elapsed_time(b) / 10
print({"d2h_bytes": x.numel() * 2, "ms": ms, "GBps": x.numel() * 2 / ms / 1e6})
PY
rm -rf /tmp/repoP; mkdir -p /tmp/repoP; cp -r . /tmp/repoP/ 2>/dev/null
cd /tmp/repoP && sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_ATTN_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py && \
  python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1
TCB_ATTN_SCHED=1 timeout 300 python scripts/attn_bench.py c2 2>&1 | grep -E "probe|workload" | tail -12 | tee $GRAFT_REPO_ROOT/$T/v3s_probe.txt
