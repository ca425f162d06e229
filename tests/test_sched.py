"""The master's task allocation core (libsw sw_sched_*, PAPER.md P18 §IV.A), on a
simulated clock.  Pinned to the paper's worked example (Fig. 5: 14 s with workload
adjustment, 18 s without) and to properties that hold for any schedule."""
import os

import numpy as np
import pytest

from paper_conf_ipps_mendoncam13_b200 import Scheduler, SW_TASK_FINISHED, SW_TASK_READY
from schedsim import simulate

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _fig5():
    grants, wa, kv = [], [], {}
    for line in open(os.path.join(GOLD, "fig5_schedule.txt")):
        if line.startswith("#") or not line.strip():
            continue
        tok = line.split()
        if tok[0] == "grant":
            grants.append((float(tok[1]), tok[2], [int(x[1:]) - 1 for x in tok[3:]]))
        elif tok[0] == "wa_grant":
            wa.append((float(tok[1]), tok[2], [int(x[1:]) - 1 for x in tok[3:]]))
        else:
            kv[tok[0]] = tok[1:]
    return grants, wa, kv


NAMES = ["GPU1", "SSE1", "SSE2", "SSE3"]


def test_fig5_with_workload_adjustment():
    grants, wa, kv = _fig5()
    speeds = [float(x) for x in kv["speeds"]]
    n = int(kv["n_tasks"][0])
    r = simulate(speeds, [6] * n, policy="pss", wa=True)
    assert r["makespan"] == pytest.approx(float(kv["makespan_wa"][0]))
    got = [(t, NAMES[w], us) for t, w, us, kind in r["grants"] if kind == "grant"]
    assert got == grants
    got_wa = [(t, NAMES[w], us) for t, w, us, kind in r["grants"] if kind == "wa"]
    assert got_wa == wa
    # t20 committed by the GPU (its replica finished first); SSE1's replica was cancelled
    assert r["commits"][19] == 0
    assert r["sched"].counter(1) == 1


def test_fig5_without_workload_adjustment():
    grants, _, kv = _fig5()
    speeds = [float(x) for x in kv["speeds"]]
    n = int(kv["n_tasks"][0])
    r = simulate(speeds, [6] * n, policy="pss", wa=False)
    assert r["makespan"] == pytest.approx(float(kv["makespan_no_wa"][0]))
    got = [(t, NAMES[w], us) for t, w, us, kind in r["grants"] if kind == "grant"]
    assert got == grants  # "the execution is exactly the same until time t13"
    assert r["commits"][19] == 1
    assert r["sched"].counter(1) == 0


def test_ss_policy_allocates_one_task():
    """SS: Allocate(N, p_i) = 1 (P18 §IV.A.1); more master interactions than PSS."""
    r_ss = simulate([6, 1, 1, 1], [6] * 20, policy="ss", wa=True)
    r_pss = simulate([6, 1, 1, 1], [6] * 20, policy="pss", wa=True)
    assert all(len(us) == 1 for _, _, us, _ in r_ss["grants"])
    assert r_ss["sched"].counter(0) > r_pss["sched"].counter(0)
    assert len(r_ss["commits"]) == 20


def test_phi_weights():
    S = Scheduler(3, [10] * 30)
    for w, v in enumerate([6.0, 1.0, 2.5]):
        S.report(w, 0.5, v * 0.5, 0.5)
    assert S.phi(0) == 6 and S.phi(1) == 1 and S.phi(2) == 3  # round half up 2.5 -> 3
    # weighted mean of the last omega reports, newest heaviest
    S2 = Scheduler(1, [10], omega=2)
    for v in (100.0, 1.0, 3.0):
        S2.report(0, 0.0, v, 1.0)
    assert S2.rate(0) == pytest.approx((1 * 1.0 + 2 * 3.0) / 3)


def test_first_allocation_one_per_slave():
    S = Scheduler(4, [5] * 12)
    for w in range(4):
        S.report(w, 0.1, 100.0 * (w + 1), 0.1)
    for w in range(4):
        assert len(S.request(w, 0.2)) == 1  # P10: "one work unit for each slave"


def test_states_and_first_result_wins():
    S = Scheduler(2, [4, 4])
    S.report(0, 0.0, 4.0, 1.0)
    S.report(1, 0.0, 1.0, 1.0)
    assert S.request(0, 0.0) == [0]
    assert S.request(1, 0.0) == [1]
    assert S.state(0) == 1 and S.replicas(1) == 1
    assert S.complete(0, 0, 1.0)
    # no ready task: WA gives worker 0 the task held by the slower worker 1
    assert S.request(0, 1.0) == [1]
    assert S.replicas(1) == 2
    assert S.complete(0, 1, 2.0) is True       # first finisher commits
    assert S.complete(1, 1, 4.0) is False      # the other replica loses
    assert S.committed_by(1) == 0 and S.state(1) == SW_TASK_FINISHED
    assert S.request(1, 4.0) is None           # all finished
    assert S.counter(2) == 4                   # duplicated cells


def test_wa_moves_a_queued_task_instead_of_duplicating():
    """A task still queued (un-started) in the holder's PSS package is moved to the idle PE
    (reading R11): one replica, the old holder's start() is refused, no duplicated cells.
    A started task (here the head of the queue) is duplicated as in Fig. 5."""
    S = Scheduler(2, [100] * 6)
    assert S.request(0, 0.0) == [0] and S.request(1, 0.0) == [1]
    S.report(0, 1.0, 300.0, 1.0)
    S.report(1, 1.0, 100.0, 1.0)
    assert S.complete(0, 0, 1.0)
    assert S.request(0, 1.0) == [2, 3, 4]              # Phi = 3
    assert S.start(0, 2, 1.0)
    assert S.complete(1, 1, 1.0)
    assert S.request(1, 1.0) == [5]
    assert S.start(1, 5, 1.0)
    S.report(0, 1.5, 10.0, 1.0)                        # worker 0 slows down (local load)
    assert S.complete(1, 5, 2.0)
    assert S.request(1, 2.0) == [4]                    # latest ETA: the tail of w0's package
    assert S.replicas(4) == 1                          # moved, not duplicated
    assert S.start(1, 4, 2.0)
    assert S.complete(1, 4, 3.0)
    assert S.request(1, 3.0) == [3]                    # next latest, also un-started
    assert S.replicas(3) == 1
    assert S.start(1, 3, 3.0) and S.complete(1, 3, 4.0)
    assert S.request(1, 4.0) == [2]                    # w0's started head: duplicated
    assert S.replicas(2) == 2
    assert S.complete(1, 2, 5.0) and not S.complete(0, 2, 9.0)
    assert not S.start(0, 3, 9.0) and not S.start(0, 4, 9.0)   # w0 skips the moved ones
    assert S.request(0, 9.0) is None
    assert S.counter(2) == 100                         # only the started head was duplicated
    assert [S.committed_by(u) for u in range(6)] == [0, 1, 1, 1, 1, 1]


def test_wa_only_when_strictly_earlier():
    S = Scheduler(2, [6])
    S.report(0, 0.0, 1.0, 1.0)
    S.report(1, 0.0, 1.0, 1.0)
    assert S.request(0, 0.0) == [0]
    assert S.request(1, 0.0) == []   # same speed started later: not strictly earlier


@pytest.mark.parametrize("seed", range(12))
def test_random_schedules_commit_every_task_once(seed):
    rng = np.random.default_rng(seed)
    n_w = int(rng.integers(1, 7))
    speeds = list(rng.uniform(0.5, 8.0, n_w))
    cells = list(rng.integers(1, 50, int(rng.integers(1, 60))))
    for policy in ("ss", "pss"):
        for wa in (True, False):
            r = simulate(speeds, cells, policy=policy, wa=wa)
            assert sorted(r["commits"]) == list(range(len(cells)))
            S = r["sched"]
            assert all(S.state(u) == SW_TASK_FINISHED for u in range(len(cells)))
            # a lower bound: total work over total speed
            assert r["makespan"] >= sum(cells) / sum(speeds) - 1e-9


def test_wa_reduces_tail_with_a_straggler():
    """One PE 6x slower (Fig. 5's ratio) holding the last tasks: WA shortens the run."""
    speeds = [6.0] * 7 + [1.0]
    cells = [6] * 41
    with_wa = simulate(speeds, cells, wa=True)["makespan"]
    without = simulate(speeds, cells, wa=False)["makespan"]
    assert with_wa < without


def test_non_dedicated_reweighting():
    """P24 §V.C: local load on one PE halves its speed; PSS lowers its package size."""
    r = simulate([2.0, 2.0, 2.0, 2.0], [1] * 400, policy="pss", wa=True,
                 slow_after=(0, 20.0, 2.5))
    S = r["sched"]
    assert S.rate(0) < S.rate(1)
    assert S.phi(1) >= 2 and S.phi(0) == 1


def test_bad_arguments():
    from paper_conf_ipps_mendoncam13_b200 import SwError
    with pytest.raises(SwError):
        Scheduler(0, [1])
    with pytest.raises(SwError):
        Scheduler(2, [1, 0])
    S = Scheduler(1, [])
    assert S.request(0, 0.0) is None


def test_failed_worker_tasks_return_to_ready():
    """R22: a worker that disappears (its connection closed) is failed: each unfinished task it
    held that nobody else runs goes back to READY and is granted before the remaining ready
    tasks; the failed worker gets nothing more, so the search completes with WA off too."""
    from paper_conf_ipps_mendoncam13_b200 import Scheduler
    S = Scheduler(2, [10, 10, 10, 10], policy="ss", wa=False)
    assert S.request(0, 0.0) == [0]
    assert S.request(1, 0.0) == [1]
    S.fail_worker(1, 0.1)
    assert S.state(1) == 0 and S.replicas(1) == 0          # READY again
    assert S.request(1, 0.2) is None                        # a failed worker gets nothing
    S.report(0, 0.3, 10, 0.1)
    assert S.complete(0, 0, 0.3)
    assert S.request(0, 0.3) == [1]                         # the re-queued task first
    for u in (1,):
        assert S.complete(0, u, 0.4)
    got = S.request(0, 0.4) + S.request(0, 0.5)
    assert sorted(got) == [2, 3]
    for u in got:
        assert S.complete(0, u, 0.6)
    assert S.request(0, 0.7) is None
    assert [e["ev"] for e in S.log()].count("F") == 1
