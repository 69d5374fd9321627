"""Independent event-driven simulator (DES) of one candidate plan.

TEST INFRASTRUCTURE ONLY.  This is the second, independently written
implementation of model M used to pin the C oracle (oracle/smiless_oracle.c)
where the paper is silent (readings G3, G4, G5, G6, G7 in DESIGN.md).  It
shares nothing with the C oracle: instead of the oracle's closed case split,
it runs an explicit per-instance state machine over timed events and bills by
integrating the time the instance is loaded.

Instance life cycle (PAPER.md:177 Case I, :188-194 Case II, :198 Case III,
:247 "timers to control the start and termination of each instance"):

* states: UNLOADED, INITIALISING (takes T), IDLE (loaded, no work), BUSY
  (serving one invocation for I; FIFO queue of waiting invocations).
* first invocation: the instance was pre-warmed to be loaded exactly when the
  first input arrives (G5): loaded from x_0 - T.
* on completion with an empty queue: window 0 -> stay IDLE (keep-alive,
  PAPER.md:194); window w > 0 -> UNLOAD now and arm a pre-warm timer at
  completion + w (reading G1).
* arrival while UNLOADED: cancel the timer, start initialising now (G3).
* arrival while INITIALISING: wait for init to finish (G4).
* billing = total time spent INITIALISING, IDLE or BUSY, ending at the last
  completion (init + inference + keep-alive cost; G7).

Events at the same timestamp are ordered arrivals first (an invocation that
arrives exactly when the previous one completes finds the instance warm, G6).
"""
from __future__ import annotations

import heapq
from typing import List, Sequence, Tuple

UNLOADED, INITIALISING, IDLE, BUSY = range(4)

# event priorities at equal time: arrivals first
_ARRIVAL, _DONE, _INIT_DONE, _PREWARM = 0, 1, 2, 3


def simulate_instance(x: Sequence[int], exec_us: int, init_us: int, window_us: int) -> Tuple[List[int], int]:
    """Serve the input-ready times x[0..J-1] (non-decreasing) on one instance.

    Returns (completion time of each invocation, billed loaded time)."""
    J = len(x)
    done = [0] * J
    ev: list = []
    seq = 0

    def push(t, kind, data=0):
        nonlocal seq
        heapq.heappush(ev, (t, kind, seq, data))
        seq += 1

    for j, t in enumerate(x):
        push(int(t), _ARRIVAL, j)

    # G5: pre-warmed so that it is loaded exactly at the first input.
    state = IDLE
    loaded_since = int(x[0]) - init_us
    billed = 0
    queue: List[int] = []
    prewarm_token = None   # (time, id) of the armed pre-warm timer
    token_id = 0
    n_done = 0

    def start_service(t):
        nonlocal state
        j = queue.pop(0)
        state = BUSY
        push(t + exec_us, _DONE, j)

    while ev:
        t, kind, _, data = heapq.heappop(ev)
        if kind == _ARRIVAL:
            queue.append(data)
            if state == IDLE:
                start_service(t)
            elif state == UNLOADED:
                prewarm_token = None                 # cancel the timer (G3)
                state = INITIALISING
                loaded_since = t
                push(t + init_us, _INIT_DONE)
            # BUSY / INITIALISING: wait in FIFO order (G4, G6)
        elif kind == _DONE:
            done[data] = t
            n_done += 1
            if n_done == J:
                billed += t - loaded_since           # billing ends at the last completion (G7)
                break
            if queue:
                start_service(t)
            elif window_us == 0:
                state = IDLE                         # keep alive (Case II)
            else:
                billed += t - loaded_since           # unload now (Case I, G1)
                state = UNLOADED
                token_id += 1
                prewarm_token = token_id
                push(t + window_us, _PREWARM, token_id)
        elif kind == _PREWARM:
            if state == UNLOADED and prewarm_token == data:
                prewarm_token = None
                state = INITIALISING
                loaded_since = t
                push(t + init_us, _INIT_DONE)
        elif kind == _INIT_DONE:
            if queue:
                start_service(t)
            else:
                state = IDLE
    return done, billed


def simulate_function(x: Sequence[int], exec_us: int, init_us: int, window_us: int,
                      instances: int = 1) -> Tuple[List[int], int]:
    """Scale-out (reading G26): `instances` identical instances, request j
    dispatched to instance j mod n (round robin), each instance serving its requests in
    request order (an input ready before the previous request of the same instance is
    admitted when that one is: effective arrival = running max over the instance's
    requests).  Returns (completion per request, billed loaded time summed over instances)."""
    J = len(x)
    done = [0] * J
    billed = 0
    for i in range(min(instances, J)):
        idx = list(range(i, J, instances))
        xs, m = [], None
        for j in idx:
            m = int(x[j]) if m is None else max(m, int(x[j]))
            xs.append(m)
        d, b = simulate_instance(xs, exec_us, init_us, window_us)
        for j, t in zip(idx, d):
            done[j] = t
        billed += b
    return done, billed


def simulate(prob, config: Sequence[int], window: Sequence[int],
             instances: Sequence[int] = None) -> Tuple[List[int], List[int]]:
    """(billed per function, E2E latency per request) for one candidate.

    Input-ready time of function k for request j: r_j for a source, else the
    latest completion among its predecessors (AND-join)."""
    n = prob.n_funcs
    r = [int(v) for v in prob.arrivals_us]
    off = [0]
    for k in range(n):
        off.append(off[-1] + int(prob.n_configs[k]))
    dones: List[List[int]] = []
    billed: List[int] = []
    listed = set()
    for k in range(n):
        preds = prob.preds(k)
        listed.update(preds)
        if not preds:
            x = list(r)
        else:
            x = [max(dones[p][j] for p in preds) for j in range(len(r))]
        row = off[k] + int(config[k])
        d, b = simulate_function(x, int(prob.exec_us[row]), int(prob.init_us[row]),
                                 int(prob.windows_us[int(window[k])]),
                                 1 if instances is None else int(instances[k]))
        dones.append(d)
        billed.append(b)
    sinks = [k for k in range(n) if k not in listed]
    lat = [max(dones[s][j] for s in sinks) - r[j] for j in range(len(r))]
    return billed, lat
