"""Run tcb_op_attention alone on a workload's packed layout with a given row count."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb
key, rows = sys.argv[1], int(sys.argv[2])
w = wl.WORKLOADS[key]
lengths, ids, _ = wl.workload_inputs(key, rows=rows)
plan = tcb.tcb_pack(lengths, w.row_len, rows)
print("rows", plan.info["num_rows"], "segments", plan.info["num_segments"], "lengths max", lengths.max(), flush=True)
M, d, h = plan.num_slots, w.model.d_model, w.model.num_heads
qkv = (torch.randn(M, 3 * d, device="cuda") * 0.5).to(torch.bfloat16)
seg = torch.from_numpy(plan.arrays()["segment_ids"]).cuda()
st = torch.from_numpy(plan.segtab()).cuda()
out = tcb.op_attention(qkv, seg, st, h)
torch.cuda.synchronize()
print("ok", float(out.float().abs().mean()), flush=True)
