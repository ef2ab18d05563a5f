"""The online serving loop (scheduler -> fixed-shape CUDA graph per time slot) on the GPU:
the responses of a scheduled batch equal the oracle's per-request outputs (the plan of
every slot is replayed through one captured graph, include/tcb.h §1 and §5)."""
import numpy as np
import pytest

import oracle
import tcb_workload as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_icpp_fuc0z22_b200 as tcb  # noqa: E402
from paper_conf_icpp_fuc0z22_b200.serve import Server  # noqa: E402
from _helpers import TOL  # noqa: E402


@pytest.mark.parametrize("policy,overlap", [("das", False), ("fcfs", False), ("das", True),
                                            ("fcfs", True)])
def test_server_responses_match_oracle(policy, overlap):
    model = wl.MODELS["toy"]
    w = wl.draw_weights(model, 3)
    names = wl.weight_names(model)
    enc = tcb.Encoder(model, w, names)
    rng = np.random.default_rng(5)
    n = 40
    lengths = rng.integers(3, 17, size=n).astype(np.int32)
    arrival = np.sort(rng.uniform(0, 0.002, size=n))
    deadline = arrival + 1.0
    offs = np.concatenate([[0], np.cumsum(lengths)])[:-1].astype(np.int64)
    ids = wl.draw_token_ids(int(lengths.sum()), model.vocab, 6)
    srv = Server(enc, policy, 2, 32, overlap=overlap)
    res = srv.run(lengths, arrival, deadline, ids, offs, horizon=10.0)
    assert res["scheduled"] == n and res["expired"] == 0 and res["batches"] >= n * 9 // 64
    got_ids, got_lens = srv.last_batch
    out = srv.last_out[:int(got_lens.sum())].float().cpu().numpy()
    base = 0
    for i, l in zip(got_ids.tolist(), got_lens.tolist()):
        tok = ids[offs[i]:offs[i] + l]
        ref = oracle.run(model, w, names, [l], tok, int(-(-l // 8) * 8))["out"]
        e = np.max(np.abs(out[base:base + l] - ref)) / np.max(np.abs(ref))
        assert e <= TOL["fp32"], (i, e)
        base += l
