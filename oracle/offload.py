"""Algorithm 1 (offload planning) and its reverse prefetch pass.
TEST INFRASTRUCTURE ONLY.  The paper prints no worked example.  Pinned (pin-12,
tests/test_offload_sim.py) by a discrete-event timeline of one FIFO copy link that knows nothing
about balances: every non-final sync finds its offloads finished (the no-stall claim)
and every prefetch not given op 0 arrives before its use; plus hand traces of both passes.
Also checked by invariants (tests/test_abi_host.py): every offloaded TSO is synchronised
(ended) no earlier than the op that started it and at the latest at the last op; the balance
is reset at every sync; offloaded bytes never exceed the theoretical limit (R15);
every prefetch starts no later than the op that needs it.

Readings:
* the candidate of op t is op t's input TSO once "no further write happens"; the
  caller passes its size (0 = not a candidate);
* loss = TSO size when offloaded; gain = t_op * BW per op;
* sync + free all TSO_to_free when balance >= 0 or at the last op; the balance is
  then reset to 0 -- also when the list is empty (no outstanding copy carries no
  capacity forward);
* the ratio cap omitted at P:275: skip an offload that would push the cumulative offloaded
  bytes above sum(t_op) * BW (the Fig. 1 limit).
"""
from __future__ import annotations


def offload_plan(op_time_s, cand_bytes, bw):
    T = len(op_time_s)
    cap = sum(t * bw for t in op_time_s)
    balance = 0.0
    offloaded = 0.0
    to_free = []
    offload = [0] * T
    sync_at = [0] * T
    for t in range(T):
        if cand_bytes[t] > 0 and offloaded + cand_bytes[t] <= cap:
            offload[t] = 1
            to_free.append(t)
            balance -= cand_bytes[t]
            offloaded += cand_bytes[t]
        balance += op_time_s[t] * bw
        if balance >= 0 or t == T - 1:
            if to_free:
                sync_at[t] = 1
            to_free = []
            balance = 0.0
    return offload, sync_at


def prefetch_plan(op_time_s, need_bytes, bw):
    """Reverse pass: walk from the last backward op to the first; a TSO needed at op t
    is a loss; each earlier op u adds t_u * BW; when the balance turns >= 0 at op u the pending
    prefetches start right before op u."""
    T = len(op_time_s)
    start = [-1] * T
    balance = 0.0
    pend = []
    for t in range(T - 1, -1, -1):
        if pend:
            balance += op_time_s[t] * bw
            if balance >= 0:
                for u in pend:
                    start[u] = t
                pend = []
                balance = 0.0
        if need_bytes[t] > 0:
            pend.append(t)
            balance -= need_bytes[t]
    for u in pend:
        start[u] = 0
    return start
