"""Host side of config 5b without a GPU: the library's async-signal-safe sink receives queued
real-time signals (rt_sigqueueinfo, the syscall the GPU issues) with their si_value intact."""
import ctypes
import os
import signal
import time

from paper_conf_isca_veselybblor18_b200 import gsys as G

SYS_rt_sigqueueinfo = 129


def _queue(sig: int, value: int) -> int:
    libc = ctypes.CDLL(None, use_errno=True)
    si = (ctypes.c_int32 * 32)()
    si[0] = sig
    si[2] = -1            # SI_QUEUE
    si[4] = os.getpid()
    si[5] = os.getuid()
    si[6] = value
    return libc.syscall(SYS_rt_sigqueueinfo, os.getpid(), sig, ctypes.byref(si))


def test_sigsink_receives_values():
    L = G.lib()
    sig = signal.SIGRTMIN + 5
    assert L.gsys_sigsink_install(sig, 256) == 0
    assert L.gsys_sigsink_install(signal.SIGUSR1, 16) < 0          # real-time signals only
    sent = list(range(100))
    for v in sent:
        assert _queue(sig, v) == 0
    got = []
    vals = (ctypes.c_int32 * 512)()
    deadline = time.time() + 5
    while len(got) < len(sent) and time.time() < deadline:
        n = L.gsys_sigsink_read(vals, None, 512)
        got += [vals[i] for i in range(n)]
    assert sorted(got) == sent


def test_sigsink_overflow_does_not_wedge_the_ring():
    """Signals that arrive while the ring is full are dropped without leaving a hole: after the
    reader drains it, later signals arrive again (the reader used to stop forever)."""
    L = G.lib()
    sig = signal.SIGRTMIN + 6
    assert L.gsys_sigsink_install(sig, 256) == 0
    vals = (ctypes.c_int32 * 1024)()
    while L.gsys_sigsink_read(vals, None, 1024) > 0:
        pass
    for v in range(300):                       # 44 more than the ring holds
        assert _queue(sig, v) == 0
    time.sleep(0.05)
    n = L.gsys_sigsink_read(vals, None, 1024)
    assert n == 256 and [vals[i] for i in range(n)] == list(range(256))
    for v in range(1000, 1010):
        assert _queue(sig, v) == 0
    got, deadline = [], time.time() + 5
    while len(got) < 10 and time.time() < deadline:
        k = L.gsys_sigsink_read(vals, None, 1024)
        got += [vals[i] for i in range(k)]
    assert got == list(range(1000, 1010))
