"""f4 measurement: greedy Seq2Seq decoding of one packed C2 batch (Transformer-base encoder +
decoder, ParaCrawl-like lengths, t_max = l_src, R32) with and without early memory cleaning
(§4.2.2, R33).  Prints one JSON line per mode: generated tokens/s (host wall clock of
tcb_decode_greedy, the whole decode incl. the encoder-memory K/V GEMMs), steps, decoder rows
computed, live KV-cache bytes (peak / mean)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb

rows = int(sys.argv[1]) if len(sys.argv) > 1 else 256
wlc = wl.WORKLOADS["c2"]
m = wlc.model
lengths = wl.lengths_filling(wlc.lengths, rows, wlc.row_len, wlc.seeds[0])
ids = wl.draw_token_ids(int(lengths.sum()), m.vocab, wlc.seeds[1])
w = wl.draw_weights(m, wlc.seeds[2])
dw = wl.draw_dec_weights(m, wlc.seeds[2] + 100)
enc = tcb.Encoder(m, w, wl.weight_names(m))
plan, enc_rows, _ = enc.run(lengths, ids, wlc.row_len, rows)
n = plan.info["num_requests"]
dec = tcb.Decoder(enc, dw, wl.dec_weight_names(m), max_requests=n, max_slots=plan.num_slots,
                  max_target=wlc.row_len)
dec.decode(plan, enc_rows, early_clean=True)           # warm-up (tensor maps, kernels)
torch.cuda.synchronize()
for clean in (True, False):
    for _ in range(2):
        t0 = time.perf_counter()
        tok, lens = dec.decode(plan, enc_rows, early_clean=clean)
        torch.cuda.synchronize()
        el = time.perf_counter() - t0
    st = dec.stats()
    print(json.dumps({"mode": "early_clean" if clean else "whole_batch", "requests": n,
                      "rows": rows, "generated_tokens": int(lens.sum()),
                      "tokens_per_s": float(lens.sum()) / el, "s": el, "steps": st["steps"],
                      "rows_computed": st["rows_computed"],
                      "kv_bytes_peak": st["kv_bytes_peak"], "kv_bytes_avg": st["kv_bytes_avg"],
                      "launches": tcb.launch_count()}), flush=True)
