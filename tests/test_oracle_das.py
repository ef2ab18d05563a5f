"""Pins of the oracle's request scheduler (§8(f) row f2) -- DESIGN.md §4.

§5: requests have arrival a_n, deadline d_n and length l_n; a batch of
B rows x L words runs per time slot; utility v_n = 1/l_n counts only for requests scheduled
inside [a_n, d_n] (Eq. (9)-(13)).  Alg. 1 (DAS) fills each row with a
utility-dominant set N_U, a deadline-aware set N_D and then the rest; Theorem 5.1 says DAS
is eta*q/(eta*q+1)-competitive (1/5 at eta = q = 1/2).

Pins: the hand-derived fixture tests/golden/f2_das.json (DAS and the FCFS/SJF/DEF
baselines); the l.4 special case; feasibility (10)-(12); greedy maximality; the N_U / N_D /
rest structure of every row read back from the outputs; equal lengths reduce DAS to
"first p in arrival order, then earliest deadline first"; and Theorem 5.1 against the
exact optimum of the MILP (9)-(13), found by exhaustive search on tiny instances.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle


def _fixture(golden_dir):
    return json.load(open(os.path.join(golden_dir, "f2_das.json")))


@pytest.mark.parametrize("case", [0, 1])
def test_f2_golden_fixture(golden_dir, case):
    c = _fixture(golden_dir)["cases"][case]
    n = len(c["lengths"])
    for pol in ("das", "fcfs", "sjf", "def"):
        if pol not in c:
            continue
        r, k = oracle.sched_batch(pol, c["lengths"], [0.0] * n, c["deadline"], range(n),
                                  c["B"], c["L"])
        assert r.tolist() == c[pol]["row"], pol
        assert k.tolist() == c[pol]["col"], pol


def _rows(r, c, lengths, B):
    out = []
    for k in range(B):
        mem = sorted([i for i in range(len(lengths)) if r[i] == k], key=lambda i: c[i])
        out.append(mem)
    return out


def _random_waiting(rng, n, L):
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    arrival = rng.integers(0, 4, size=n).astype(np.float64)     # ties exercised
    deadline = arrival + rng.integers(0, 6, size=n)
    ids = rng.permutation(1000)[:n].astype(np.int64)
    return lengths, arrival, deadline, ids


@pytest.mark.parametrize("policy", ["das", "fcfs", "sjf", "def"])
@pytest.mark.parametrize("seed", range(25))
def test_feasible_contiguous_and_greedy_maximal(policy, seed):
    rng = np.random.default_rng(9100 + seed)
    L = int(rng.choice([8, 16, 64]))
    B = int(rng.integers(1, 5))
    n = int(rng.integers(0, 30))
    lengths, arrival, deadline, ids = _random_waiting(rng, n, L)
    r, c = oracle.sched_batch(policy, lengths, arrival, deadline, ids, B, L)
    rows = _rows(r, c, lengths, B)
    placed_before = set()
    for k, mem in enumerate(rows):
        used = 0
        for i in mem:                       # contiguous from column 0, constraint (11)
            assert c[i] == used
            used += int(lengths[i])
        assert used <= L
        placed_before |= set(mem)
        # greedy maximality: nothing left after row k fits its residual
        for i in range(n):
            if i not in placed_before:
                assert lengths[i] > L - used, (k, i)
    assert all((r[i] < 0) == (c[i] < 0) for i in range(n))       # constraint (10) by shape


@pytest.mark.parametrize("seed", range(40))
def test_das_row_structure(seed):
    """Each row = N_U (the p highest-utility of what is left, p = max(1, floor(eta s)))
    then N_D members (v >= q * mean v(N_U)) in deadline order, then the rest in utility
    order -- or, when everything left fits, everything left in arrival order."""
    rng = np.random.default_rng(9300 + seed)
    L = int(rng.choice([8, 16, 64]))
    B = int(rng.integers(1, 5))
    n = int(rng.integers(1, 30))
    eta = float(rng.choice([0.5, 0.3, 0.7]))
    q = 1.0 - eta
    lengths, arrival, deadline, ids = _random_waiting(rng, n, L)
    r, c = oracle.sched_batch("das", lengths, arrival, deadline, ids, B, L, eta, q)
    left = list(range(n))
    util_key = lambda i: (lengths[i], arrival[i], ids[i])
    for mem in _rows(r, c, lengths, B):
        if not left:
            assert not mem
            continue
        if sum(int(lengths[i]) for i in left) <= L:
            assert mem == sorted(left, key=lambda i: (arrival[i], ids[i]))
            left = []
            continue
        seq = sorted(left, key=util_key)
        pre, s = 0, 0
        while s < len(seq) and pre + lengths[seq[s]] <= L:
            pre += int(lengths[seq[s]])
            s += 1
        p = max(1, math.floor(eta * s))
        assert mem[:p] == seq[:p]
        vbar = sum(1.0 / lengths[i] for i in seq[:p]) / p
        tail = mem[p:]
        nd = [i for i in tail if 1.0 / lengths[i] >= q * vbar]
        rest = [i for i in tail if 1.0 / lengths[i] < q * vbar]
        assert tail == nd + rest
        assert nd == sorted(nd, key=lambda i: (deadline[i], arrival[i], ids[i]))
        assert rest == sorted(rest, key=util_key)
        left = [i for i in left if i not in mem]


def test_das_all_fit_one_row_and_equal_lengths():
    # l.4-5: everything fits row 0 -> all of it, arrival order, other rows empty
    r, c = oracle.sched_batch("das", [3, 2, 1], [2.0, 0.0, 1.0], [9, 9, 9], [0, 1, 2], 3, 8)
    assert r.tolist() == [0, 0, 0] and c.tolist() == [3, 0, 2]
    # equal lengths: N_U = first p in arrival order, N_D = everyone else -> EDF
    n, l, L = 9, 4, 16                     # s = 4, p = 2 per row
    deadline = [7, 3, 5, 1, 8, 2, 6, 4, 0]
    r, c = oracle.sched_batch("das", [l] * n, [0.0] * n, deadline, range(n), 2, L)
    rows = _rows(r, c, [l] * n, 2)
    assert rows[0] == [0, 1, 8, 3]          # r0, r1 (arrival) then d=0 (r8), d=1 (r3)
    assert rows[1] == [2, 4, 5, 7]          # r2, r4 (arrival) then d=2 (r5), d=4 (r7)


def _opt_bruteforce(lengths, arrival, deadline, B, L, T, slot_time):
    """Exact optimum of (9)-(13): each request goes to one (slot, row) inside its window
    or nowhere; row loads <= L.  Depth-first over requests with capacity pruning."""
    n = len(lengths)
    v = [1.0 / l for l in lengths]
    opts = []
    for i in range(n):
        o = [(t, k) for t in range(T) for k in range(B)
             if arrival[i] <= t * slot_time <= deadline[i]]
        opts.append(o)
    load = {}
    best = [0.0]
    order = sorted(range(n), key=lambda i: -v[i])
    suffix = [0.0] * (n + 1)
    for j in range(n - 1, -1, -1):
        suffix[j] = suffix[j + 1] + v[order[j]]

    def rec(j, val):
        if val + suffix[j] <= best[0] + 1e-15:
            return
        if j == n:
            best[0] = val
            return
        i = order[j]
        for tk in opts[i]:
            if load.get(tk, 0) + lengths[i] <= L:
                load[tk] = load.get(tk, 0) + lengths[i]
                rec(j + 1, val + v[i])
                load[tk] -= lengths[i]
        rec(j + 1, val)

    rec(0, 0.0)
    return best[0]


@pytest.mark.parametrize("eta", [0.5, 0.3, 0.7])
@pytest.mark.parametrize("seed", range(40))
def test_theorem_5_1_competitive_ratio(eta, seed):
    """ALG >= eta*q/(eta*q + 1) * OPT with q = 1 - eta (Theorem 5.1)
    on random tiny online instances; OPT by exhaustive search of the MILP (9)-(13)."""
    q = 1.0 - eta
    rng = np.random.default_rng(9500 + seed)
    n = int(rng.integers(2, 8))
    L = int(rng.choice([4, 6, 8]))
    B = int(rng.integers(1, 3))
    T = int(rng.integers(1, 4))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    arrival = rng.integers(0, T, size=n).astype(np.float64)
    deadline = arrival + rng.integers(0, 3, size=n)
    alg = oracle.sched_simulate("das", lengths, arrival, deadline, B, L, 1.0, T, eta, q)
    opt = _opt_bruteforce(lengths.tolist(), arrival, deadline, B, L, T, 1.0)
    # ALG itself is feasible for (10)-(12)
    for i in range(n):
        if alg["slot"][i] >= 0:
            assert arrival[i] <= alg["slot"][i] <= deadline[i]
    assert alg["utility"] <= opt + 1e-12
    assert alg["utility"] >= eta * q / (eta * q + 1) * opt - 1e-12, (alg["utility"], opt)


def test_sched_errors():
    with pytest.raises(oracle.OracleError) as e:
        oracle.sched_batch("das", [3, 9], [0, 0], [1, 1], [0, 1], 1, 8)
    assert e.value.code == -2
    r, c = oracle.sched_batch("das", [], [], [], [], 2, 8)
    assert len(r) == 0
