"""ThreadSanitizer on the master's task-allocation core: tools/sched_tsan.cpp
drives one sw_sched from 6 worker threads the way libsw's workers do (long-poll requests,
start, progress reports, first-result-wins completion, abandoning WA replicas, one 6x slower
worker, one worker failing mid-run) under SS/PSS x WA off/on; every task must be committed
exactly once and TSan must report nothing.  CPU only."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_scheduler_core_is_race_free(tmp_path):
    gxx = shutil.which("g++")
    if gxx is None:
        pytest.skip("no g++")
    exe = str(tmp_path / "sched_tsan")
    src = [os.path.join(ROOT, "tools", "sched_tsan.cpp"),
           os.path.join(ROOT, "paper_conf_ipps_mendoncam13_b200", "csrc", "sched.cpp")]
    b = subprocess.run([gxx, "-std=c++17", "-O1", "-g", "-fsanitize=thread", "-pthread", *src, "-o", exe],
                       capture_output=True, text=True)
    if b.returncode != 0 and "fsanitize" in b.stderr:
        pytest.skip("ThreadSanitizer unavailable: " + b.stderr[-200:])
    assert b.returncode == 0, b.stderr[-2000:]
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300,
                       env=dict(os.environ, TSAN_OPTIONS="halt_on_error=1 exitcode=66"))
    out = r.stdout + r.stderr
    assert r.returncode == 0, out[-3000:]
    assert "sched tsan ok" in r.stdout
    assert "ThreadSanitizer" not in out, out[-3000:]
