"""CPU tests of the C++ request scheduler (include/tcb.h §5, §8(f) row f2) against the
oracle's scheduler (oracle_sched_batch, pinned in test_oracle_das.py): bit-exact batch
decisions for DAS / FCFS / SJF / DEF on random waiting sets and the golden fixture F2; the
stateful online loop (tcb_sched_submit / tcb_sched_next_batch) against the oracle's online
simulation slot by slot; the batch plans it emits; error conventions.
"""
import json
import os

import numpy as np
import pytest

import oracle
import paper_conf_icpp_fuc0z22_b200 as tcb


def _waiting(rng, n, L, arrivals=4, slack=6, len_hi=None):
    lengths = rng.integers(1, (len_hi or L) + 1, size=n).astype(np.int32)
    arrival = rng.integers(0, arrivals, size=n).astype(np.float64)
    deadline = arrival + rng.integers(0, slack, size=n)
    ids = rng.permutation(10 * n + 10)[:n].astype(np.int64)
    return lengths, arrival, deadline, ids


@pytest.mark.parametrize("policy", ["das", "fcfs", "sjf", "def"])
@pytest.mark.parametrize("seed", range(30))
def test_sched_batch_bit_exact_vs_oracle(policy, seed):
    rng = np.random.default_rng(9700 + seed)
    L = int(rng.choice([8, 16, 64, 128, 256]))
    B = int(rng.integers(1, 17))
    n = int(rng.integers(0, 400))
    eta = float(rng.choice([0.5, 0.3, 0.7, 0.25]))
    q = 1.0 - eta
    lengths, arrival, deadline, ids = _waiting(rng, n, L, len_hi=int(rng.choice([L, max(1, L // 4)])))
    a = tcb.sched_batch(policy, lengths, arrival, deadline, ids, B, L, eta, q)
    o = oracle.sched_batch(policy, lengths, arrival, deadline, ids, B, L, eta, q)
    assert a[0].tolist() == o[0].tolist()
    assert a[1].tolist() == o[1].tolist()


def test_sched_batch_golden_f2(golden_dir):
    f = json.load(open(os.path.join(golden_dir, "f2_das.json")))
    for c in f["cases"]:
        n = len(c["lengths"])
        for pol in ("das", "fcfs", "sjf", "def"):
            if pol in c:
                r, k = tcb.sched_batch(pol, c["lengths"], [0.0] * n, c["deadline"], range(n),
                                       c["B"], c["L"])
                assert r.tolist() == c[pol]["row"] and k.tolist() == c[pol]["col"], pol


@pytest.mark.parametrize("policy", ["das", "fcfs", "sjf", "def"])
@pytest.mark.parametrize("seed", range(8))
def test_online_loop_matches_oracle_simulation(policy, seed):
    rng = np.random.default_rng(9900 + seed)
    L, B, T = 32, 3, 12
    n = 120
    lengths = np.minimum(np.rint(rng.normal(8, 3, size=n)), L).clip(1).astype(np.int32)
    arrival = np.sort(rng.uniform(0, T * 0.7, size=n))
    deadline = arrival + rng.uniform(0.5, 4.0, size=n)
    ids = np.arange(n, dtype=np.int64)
    ref = oracle.sched_simulate(policy, lengths, arrival, deadline, B, L, 1.0, T)
    s = tcb.Scheduler(policy, B, L)
    s.submit(ids, lengths, arrival, deadline)
    slot = np.full(n, -1)
    row = np.full(n, -1)
    col = np.full(n, -1)
    for t in range(T):
        got, lens, plan = s.next_batch(float(t))
        assert plan.info["num_rows"] == B and plan.info["row_len"] == L
        a = plan.arrays()
        assert lens.tolist() == lengths[got].tolist()
        for j, i in enumerate(got):
            slot[i], row[i], col[i] = t, a["req_row"][j], a["req_col"][j]
        # (row, column) order of the output
        keys = list(zip(a["req_row"].tolist(), a["req_col"].tolist()))
        assert keys == sorted(keys)
    assert slot.tolist() == ref["slot"].tolist()
    assert row.tolist() == ref["row"].tolist()
    assert col.tolist() == ref["col"].tolist()
    st = s.stats()
    assert st["submitted"] == n and st["scheduled"] == int((slot >= 0).sum())
    assert st["batches"] == T
    assert st["utility"] == pytest.approx(ref["utility"], rel=1e-12)
    # every request is scheduled, expired, or still waiting (not yet expired at the end)
    assert st["scheduled"] + st["expired"] + st["waiting"] == n


def test_plan_of_a_batch_runs_the_layout_rules():
    s = tcb.Scheduler("das", 4, 16)
    s.submit([10, 11, 12], [5, 7, 3], [0.0, 0.0, 0.0], [9.0, 9.0, 9.0])
    ids, lens, plan = s.next_batch(0.0)
    assert sorted(ids.tolist()) == [10, 11, 12]
    assert plan.info["num_rows"] == 4 and plan.info["num_slots"] == 64
    a = plan.arrays()
    # l.4-5: everything fits row 0 in arrival order (ties by id)
    assert ids.tolist() == [10, 11, 12] and a["req_col"].tolist() == [0, 5, 12]
    assert (a["segment_ids"][16:] == -1).all()
    st = plan.segtab()
    assert st[:4].tolist() == [3, 64, 16, 15]
    ids, lens, plan = s.next_batch(1.0)
    assert len(ids) == 0 and plan.info["num_segments"] == 0


def test_expiry_and_future_arrivals():
    s = tcb.Scheduler("fcfs", 1, 8)
    s.submit([1, 2, 3], [8, 8, 8], [0.0, 0.0, 5.0], [0.5, 3.0, 9.0])
    ids, _, _ = s.next_batch(0.0)
    assert ids.tolist() == [1]
    ids, _, _ = s.next_batch(4.0)            # request 2 expired at 3.0; 3 arrives at 5.0
    assert ids.tolist() == []
    ids, _, _ = s.next_batch(5.0)
    assert ids.tolist() == [3]
    st = s.stats()
    assert st["expired"] == 1 and st["scheduled"] == 2 and st["waiting"] == 0


def test_sched_errors():
    with pytest.raises(tcb.TcbError) as e:
        tcb.sched_batch("das", [3, 9], [0, 0], [1, 1], [0, 1], 1, 8)
    assert e.value.status == -2
    with pytest.raises(tcb.TcbError):
        tcb.sched_batch("das", [3], [0], [1], [0], 1, 8, eta=0.0)
    with pytest.raises(tcb.TcbError):
        tcb.Scheduler("das", 0, 8)
    with pytest.raises(tcb.TcbError):
        tcb.Scheduler("das", 2, 12)          # row_len % 8 != 0
    s = tcb.Scheduler("das", 2, 8)
    with pytest.raises(tcb.TcbError) as e:
        s.submit([1], [9], [0.0], [1.0])
    assert e.value.status == -2
    with pytest.raises(tcb.TcbError):
        s.submit([1], [3], [2.0], [1.0])     # deadline < arrival
    assert s.stats()["submitted"] == 0
