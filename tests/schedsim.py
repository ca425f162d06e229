"""Discrete-event simulation of master + slaves on a simulated clock, driving libsw's
task-allocation core (sw_sched_*) exactly as the GPU workers do (request when idle,
progress notifications, complete -> commit or lose, cancel losing replicas)."""
import heapq

from paper_conf_ipps_mendoncam13_b200 import Scheduler


def simulate(speeds, unit_cells, policy="pss", wa=True, omega=4, heartbeat=0.5, slow_after=None,
             t_end=1e9):
    """speeds[w] = cells/s of worker w.  slow_after = (worker, time, factor): the worker's
    speed drops by `factor` from `time` on (non-dedicated PE, P24 §V.C).
    Returns dict(makespan, grants=[(t, w, [units], kind)], commits={u: w}, finish={w: t})."""
    S = Scheduler(len(speeds), unit_cells, policy=policy, wa=wa, omega=omega)
    n = len(speeds)
    speed = list(map(float, speeds))
    queue = [[] for _ in range(n)]          # tasks granted, in order
    current = [None] * n                    # (unit, start, end)
    grants, commits, finish = [], {}, {}
    ev = []                                 # (time, seq, kind, worker, payload)
    seq = [0]

    def push(t, kind, w, payload=None):
        seq[0] += 1
        heapq.heappush(ev, (t, seq[0], kind, w, payload))

    def start_next(w, t):
        while queue[w]:
            u = queue[w].pop(0)
            if not S.start(w, u, t):   # finished elsewhere or moved away by WA
                continue
            dur = unit_cells[u] / speed[w]
            current[w] = (u, t, t + dur)
            push(t + dur, "done", w, u)
            return True
        current[w] = None
        return False

    def ask(w, t):
        got = S.request(w, t)
        if got is None:
            return False
        if got:
            kind = "wa" if (len(got) == 1 and any(got[0] in g[2] for g in grants)) else "grant"
            grants.append((t, w, got, kind))
            queue[w].extend(got)
            start_next(w, t)
            return True
        return False

    t = 0.0
    for w in range(n):
        ask(w, 0.0)
        push(heartbeat, "hb", w)
    done_all = False
    while ev and not done_all:
        t, _, kind, w, payload = heapq.heappop(ev)
        if t > t_end:
            break
        if slow_after and w == slow_after[0] and t >= slow_after[1] and speed[w] == speeds[w]:
            speed[w] = speeds[w] / slow_after[2]
        if kind == "hb":
            if current[w] is not None:
                S.report(w, t, speed[w] * heartbeat, heartbeat)
            push(t + heartbeat, "hb", w)
            continue
        if kind == "done":
            if current[w] is None or current[w][0] != payload or abs(current[w][2] - t) > 1e-9:
                continue  # stale (cancelled)
            u = payload
            if S.complete(w, u, t):
                commits[u] = w
                finish[w] = t
                # cancel the other replica(s)
                for v in range(n):
                    if v != w and current[v] is not None and current[v][0] == u:
                        S.abandon(v, u, t)
                        current[v] = None
                        if not start_next(v, t):
                            ask(v, t)
            if not start_next(w, t):
                ask(w, t)
            if len(commits) == len(unit_cells):
                done_all = True
                break
        # idle workers poll the master at every event (a request costs nothing here)
        for v in range(n):
            if current[v] is None and not queue[v]:
                ask(v, t)
    return dict(makespan=t, grants=grants, commits=commits, finish=finish, sched=S)
