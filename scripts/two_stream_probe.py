"""Experiment: does running the batch as two independent row halves on two streams (one CUDA
graph with a fork / join) beat one full-batch forward?  Rows never interact, so the halves
share nothing; the question is whether one half's kernels fill the other's tails.
Run with TCB_LN_KERNEL=cluster (the L2-exchange LN kernel assumes a co-resident grid and must
not run concurrently with itself)."""
import json, os, sys
os.environ.setdefault("TCB_LN_KERNEL", "cluster")   # never two L2-exchange kernels at once
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb

key = sys.argv[1] if len(sys.argv) > 1 else "c2"
w = wl.WORKLOADS[key]
m = w.model
names = wl.weight_names(m)
weights = wl.draw_weights(m, w.seeds[2])
base = tcb.Encoder(m, weights, names)
views = [base._tensors[i] for i in range(len(names))] if hasattr(base, "_tensors") else None
encs = [tcb.Encoder(m, weights, names) for _ in range(2)]
dev = torch.device("cuda")
flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)


def prep(enc, rows, seed):
    lengths = wl.lengths_filling(w.lengths, rows, w.row_len, seed)
    ids = wl.draw_token_ids(int(lengths.sum()), m.vocab, seed + 1)
    plan = tcb.tcb_pack(lengths, w.row_len, rows)
    seg = torch.from_numpy(plan.segtab()).to(dev)
    d_ids = torch.from_numpy(ids).to(dev)
    out_rows = enc.alloc_rows(plan.num_slots)
    enc.workspace(plan.num_slots)
    return plan, seg, d_ids, out_rows, int(plan.info["placed_tokens"])


def timed(g, it=20):
    ts = []
    for _ in range(it):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); g.replay(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return float(np.median(ts))


s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
# one full batch
full = prep(base, w.rows, w.seeds[0])
for _ in range(2):
    base.encoder_forward(full[0], full[1], full[2], full[3], stream=s0)
torch.cuda.synchronize()
g_full = torch.cuda.CUDAGraph()
with torch.cuda.graph(g_full, stream=s0):
    base.encoder_forward(full[0], full[1], full[2], full[3], stream=s0)
ms_full = timed(g_full)
# two halves on two streams
halves = [prep(encs[i], w.rows // 2, w.seeds[0] + 17 * (i + 1)) for i in range(2)]
for _ in range(2):
    for i, s in enumerate((s0, s1)):
        encs[i].encoder_forward(halves[i][0], halves[i][1], halves[i][2], halves[i][3], stream=s)
torch.cuda.synchronize()
g2 = torch.cuda.CUDAGraph()
with torch.cuda.graph(g2, stream=s0):
    s1.wait_stream(s0)
    encs[0].encoder_forward(halves[0][0], halves[0][1], halves[0][2], halves[0][3], stream=s0)
    with torch.cuda.stream(s1):
        encs[1].encoder_forward(halves[1][0], halves[1][1], halves[1][2], halves[1][3], stream=s1)
    s0.wait_stream(s1)
ms_two = timed(g2)
# the two halves one after the other on one stream (same kernels, no concurrency)
g_seq = torch.cuda.CUDAGraph()
with torch.cuda.graph(g_seq, stream=s0):
    for i in range(2):
        encs[i].encoder_forward(halves[i][0], halves[i][1], halves[i][2], halves[i][3], stream=s0)
ms_seq = timed(g_seq)
tok_full = full[4]
tok_two = halves[0][4] + halves[1][4]
print(json.dumps({"workload": key, "ln_kernel": os.environ.get("TCB_LN_KERNEL", "default"),
                  "full_ms": ms_full, "full_tok_s": tok_full / ms_full * 1e3,
                  "two_stream_ms": ms_two, "two_stream_tok_s": tok_two / ms_two * 1e3,
                  "halves_serial_ms": ms_seq, "halves_serial_tok_s": tok_two / ms_seq * 1e3}))
