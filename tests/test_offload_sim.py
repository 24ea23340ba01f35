"""Pin-12: Algorithm 1 and its reverse prefetch pass against a discrete-event
timeline of one copy link, independent of the planners' balance arithmetic.

The paper's claim is the property being pinned: offloads are synchronised only when the balance
is >= 0, "so there will be no outstanding memory transfer" at the sync, i.e. compute
never waits on a copy.  The simulator below knows nothing about balances: ops run back to back
(op t occupies [T_t, T_t + t_op)); a copy is queued on ONE FIFO link of bandwidth BW when it is
issued and takes bytes / BW once the link is free.

* offload (forward order): the D2H of op t's input TSO is issued at the start of op t (no write
  after that point); every TSO in a sync list must have finished by the end of the sync op
  -- except the forced sync at the last op, which may wait.
* prefetch (backward order): the H2D of the TSO needed by op t is issued at the start of
  the op the pass chose; copies issued together go in ascending order of use; every prefetch must
  have finished by the start of the op that needs it -- TSOs given op 0 (which include the
  leftovers the pass could not cover) are treated as resident before the backward pass begins.

Plus a small hand-worked case of each pass, traced from the algorithm's lines by hand.
"""
import random

import pytest

from oracle import offload as OO

EPS = 1e-9


def _starts(times):
    s, acc = [], 0.0
    for t in times:
        s.append(acc)
        acc += t
    return s


def _link(issues, bw):
    """issues: list of (issue_time, order_key, bytes, tag); FIFO by (issue_time, order_key).
    Returns {tag: finish_time}."""
    free, done = 0.0, {}
    for t0, _, nbytes, tag in sorted(issues, key=lambda e: (e[0], e[1])):
        begin = max(free, t0)
        free = begin + nbytes / bw
        done[tag] = free
    return done


def _random_case(rng, T):
    times = [rng.choice([0.0, rng.uniform(0.01, 2.0)]) if rng.random() < 0.2 else rng.uniform(0.01, 2.0)
             for _ in range(T)]
    bw = rng.uniform(0.5, 4.0)
    cand = [0 if rng.random() < 0.3 else rng.randint(1, 12) for _ in range(T)]
    return times, cand, bw


@pytest.mark.parametrize("seed", range(40))
def test_offload_syncs_never_wait_on_the_link(seed):
    rng = random.Random(1000 + seed)
    T = rng.randint(1, 30)
    times, cand, bw = _random_case(rng, T)
    off, sync = OO.offload_plan(times, cand, bw)
    start = _starts(times)
    done = _link([(start[t], t, cand[t], t) for t in range(T) if off[t]], bw)
    pending = []
    for t in range(T):
        if off[t]:
            pending.append(t)
        if sync[t]:
            end_t = start[t] + times[t]
            if t != T - 1:
                for u in pending:
                    assert done[u] <= end_t + EPS, (t, u, done[u], end_t)
            pending = []
    assert not pending                         # every offloaded TSO is in some sync list


@pytest.mark.parametrize("seed", range(40))
def test_prefetches_arrive_before_use(seed):
    rng = random.Random(2000 + seed)
    T = rng.randint(1, 30)
    times, need, bw = _random_case(rng, T)
    st = OO.prefetch_plan(times, need, bw)
    start = _starts(times)
    for t in range(T):
        if need[t] > 0:
            assert 0 <= st[t] < t or (st[t] == 0 and t == 0)
    # TSOs given op 0 include the leftovers the pass could not cover (it ran out of ops);
    # they may stall, so the timeline treats them as resident before the backward pass begins and
    # checks that every other prefetch arrives before its use
    issues = [(start[st[t]], t, need[t], t) for t in range(T) if need[t] > 0 and st[t] > 0]
    done = _link(issues, bw)
    for t, fin in done.items():
        assert fin <= start[t] + EPS, (t, st[t], fin, start[t])


def test_offload_hand_trace():
    # BW = 1 byte/s, four 1-s ops, TSOs of 3 and 1 bytes at ops 0 and 3; cap = 4 bytes.
    # op0: offload 3 (0+3 <= 4), balance -3+1 = -2; op1: -1; op2: 0 >= 0 -> sync {0}, reset;
    # op3: offload 1 (3+1 <= 4), balance -1+1 = 0 -> sync {3}.
    assert OO.offload_plan([1.0] * 4, [3, 0, 0, 1], 1.0) == ([1, 0, 0, 1], [0, 0, 1, 1])
    # the cap skips an offload: 3 + 2 > 4 at op 3, so op 3 is not offloaded and has no sync
    assert OO.offload_plan([1.0] * 4, [3, 0, 0, 2], 1.0) == ([1, 0, 0, 0], [0, 0, 1, 0])


def test_prefetch_hand_trace():
    # BW = 1, four 1-s backward ops; op 3 needs 2 bytes, op 1 needs 1 byte.
    # t=3: append 3 (balance -2); t=2: -1; t=1: 0 >= 0 -> start 3 before op 1, reset; append 1 (-1);
    # t=0: 0 >= 0 -> start 1 before op 0.
    assert OO.prefetch_plan([1.0] * 4, [0, 1, 0, 2], 1.0) == [-1, 0, -1, 1]
