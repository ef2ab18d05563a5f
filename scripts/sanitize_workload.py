"""A small workload for compute-sanitizer (memcheck / racecheck / synccheck): every kernel of
the forward path on tiny shapes -- the fp32 toy encoder (SIMT path) and a 2-layer bf16
encoder per d in {512, 768, 1024} (tcgen05 GEMMs incl. the LN-fused cluster and L2-exchange
kernels, attention, pack_embed, unpack) -- plus the greedy decoder for d = 512.
Exit code 0 iff every call succeeded; the sanitizer reports memory / race / sync errors."""
import dataclasses
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import tcb_workload as wl  # noqa: E402
import paper_conf_icpp_fuc0z22_b200 as tcb  # noqa: E402


def run(model, lengths, row_len, rows, decode=False):
    names = wl.weight_names(model)
    w = wl.draw_weights(model, 3)
    enc = tcb.Encoder(model, w, names)
    ids = wl.draw_token_ids(int(np.sum(lengths)), model.vocab, 4)
    plan, out_rows, out = enc.run(np.asarray(lengths, np.int32), ids, row_len, rows)
    torch.cuda.synchronize()
    assert torch.isfinite(out.float()).all()
    if decode:
        dw = wl.draw_dec_weights(model, 5)
        dec = tcb.Decoder(enc, dw, wl.dec_weight_names(model), max_requests=len(lengths),
                          max_slots=plan.num_slots, max_target=8)
        dec.decode(plan, out_rows, early_clean=True)
        torch.cuda.synchronize()
    print(model.name, model.d_model, "ok", flush=True)


toy = wl.MODELS["toy"]
run(toy, [14, 11, 10, 6, 7, 3, 4, 3], 32, 2)
base = wl.MODELS["transformer-base"]
for d, h in ((512, 8), (768, 12), (1024, 16)):
    m = dataclasses.replace(base, num_layers=2, d_model=d, num_heads=h, d_ff=4 * d, vocab=512)
    # 2 rows of 128: several requests per row, a tail of padding, a pad-only q-block tile
    run(m, [30, 41, 17, 25, 60, 9, 33], 128, 2, decode=(d == 512))
print("sanitize workload done", flush=True)
