"""CPU tests of the persistent server's host state machine (runtime.cu) against
an emulated ring device (algas_server_create_emulated): a host thread that
follows the persistent kernel's side of the ring protocol -- READY/epoch
pickup per slot, two ring entries per slot served alternately, per-CTA lists
+ Finish words -- so slot claims, staging ahead, epochs, the poller's merge
and recycle, the FIFO drain, the watchdog and bounded sessions run without a
GPU (P:L166-172 states, P:L221-223 host merge, P:L261 single writer per word).

The emulated device's lists are a fixed function of the query (not a search):
the merged result of query tag t is ids t*1000 + j, dists q[0] + j, j < k,
after the host merge dropped the repeated id CTA 1 adds for T > 1.
"""
import threading
import time

import numpy as np
import pytest

import paper_conf_ipps_chencyzw025_b200 as algas

SENT = 0xFFFFFFFF


def _params(slots, T, k=10, host_threads=1, watchdog_ms=0):
    return algas.default_params(k=k, itopk=max(16, k), width=4, ctas_per_query=T, slots=slots,
                                host_threads=host_threads, watchdog_ms=watchdog_ms)


def _queries(n, dim=8, seed=0):
    rng = np.random.default_rng(seed)
    Q = rng.integers(0, 1000, size=(n, dim)).astype(np.float32)
    return np.ascontiguousarray(Q)


def _drain(srv, n, timeout=20.0):
    got = {}
    t0 = time.time()
    while len(got) < n and time.time() - t0 < timeout:
        tags, ids, ds, st = srv.poll(128)
        for t, i, d in zip(tags, ids, ds):
            assert int(t) not in got, f"tag {int(t)} returned twice"
            got[int(t)] = (i.copy(), d.copy())
        if len(tags) == 0:
            time.sleep(0.0005)
    return got


def _expect(tag, q0, k, kmax):
    ids = np.full(kmax, SENT, np.uint32)
    ds = np.full(kmax, np.inf, np.float32)
    ids[:k] = tag * 1000 + np.arange(k)
    ds[:k] = q0 + np.arange(k, dtype=np.float32)
    return ids, ds


@pytest.mark.parametrize("slots,T,host_threads", [(1, 1, 1), (3, 2, 1), (32, 4, 1), (8, 4, 2), (5, 3, 3)])
def test_fifo_every_query_once_with_its_own_result(slots, T, host_threads):
    """enqueue -> poller feeds free entries -> device -> Finish -> host merge
    -> completion queue: every tag comes back exactly once with ITS query's
    result (the merge of its T lists, duplicates dropped)."""
    n = 600
    Q = _queries(n, seed=slots)
    with algas.Server(None, _params(slots, T, host_threads=host_threads), emulated_dim=8) as srv:
        srv.enqueue(Q, tag0=7)
        got = _drain(srv, n)
        assert len(got) == n
        for i in range(n):
            ei, ed = _expect(7 + i, Q[i, 0], 10, 10)
            gi, gd = got[7 + i]
            np.testing.assert_array_equal(gi, ei)
            np.testing.assert_array_equal(gd, ed)
        assert srv.inflight() == 0


def test_ring_capacity_is_two_entries_per_slot_then_start():
    """Before the device runs, submit stages up to two queries per slot
    (None -> Work for both ring entries) and then refuses (EAGAIN);
    once started, every staged query completes."""
    slots, T = 4, 2
    Q = _queries(20)
    with algas.Server(None, _params(slots, T), deferred=True, emulated_dim=8) as srv:
        acc = [srv.submit(Q[i], tag=i) for i in range(20)]
        assert sum(acc) == 2 * slots and all(acc[:2 * slots]) and not any(acc[2 * slots:])
        srv.start()
        got = _drain(srv, 2 * slots)
        assert sorted(got) == list(range(2 * slots))
        for t in got:
            np.testing.assert_array_equal(got[t][0], _expect(t, Q[t, 0], 10, 10)[0])


def test_bounded_session_drains_staged_queries_and_refuses_new_work():
    slots, T = 3, 4
    Q = _queries(6)
    with algas.Server(None, _params(slots, T), deferred=True, emulated_dim=8) as srv:
        n = srv.submit_many(Q, tag0=50)
        assert n == 6
        srv.start(quit_when_idle=True)
        got = _drain(srv, 6)
        assert sorted(got) == list(range(50, 56))
        with pytest.raises(algas.AlgasError):
            srv.submit(Q[0], tag=99)


def test_smaller_per_query_k_pads_with_sentinels():
    Q = _queries(10)
    with algas.Server(None, _params(4, 2, k=10), emulated_dim=8) as srv:
        for i in range(10):
            while not srv.submit(Q[i], tag=i, k=4):
                time.sleep(0.0005)
        got = _drain(srv, 10)
        for t in range(10):
            ei, ed = _expect(t, Q[t, 0], 4, 10)
            np.testing.assert_array_equal(got[t][0], ei)
            np.testing.assert_array_equal(got[t][1], ed)


def test_submit_rejects_work_beyond_server_limits():
    with algas.Server(None, _params(2, 1, k=10), emulated_dim=8) as srv:
        q = _queries(1)[0]
        for kw in (dict(k=11), dict(itopk=64), dict(width=33)):
            with pytest.raises(algas.AlgasError):
                srv.submit(q, tag=1, **kw)


def test_watchdog_reports_a_query_stuck_in_its_slot():
    """A query the device never finishes is reported by algas_poll after
    watchdog_ms (no silent wait); the other slots keep serving."""
    Q = _queries(40)
    with algas.Server(None, _params(4, 2, watchdog_ms=150), emulated_dim=8) as srv:
        srv.emulated_stall(13)
        srv.enqueue(Q, tag0=0)
        seen = set()
        err = None
        t0 = time.time()
        while time.time() - t0 < 10:
            try:
                tags, _, _, _ = srv.poll(64)
                seen.update(int(t) for t in tags)
            except algas.AlgasError as e:
                err = e
                break
            time.sleep(0.001)
        # (the stalled query, or the one staged behind it in the same slot's
        # other ring entry -- both are stuck in that slot)
        assert err is not None and "watchdog" in str(err), err
        assert 13 not in seen and len(seen) > 0


def test_concurrent_producers_and_consumer():
    """Two producer threads enqueue while the caller polls: no tag lost or
    duplicated (ctypes releases the GIL around every library call)."""
    n_each = 400
    Qa, Qb = _queries(n_each, seed=1), _queries(n_each, seed=2)
    with algas.Server(None, _params(6, 4, host_threads=2), emulated_dim=8) as srv:
        def prod(Q, tag0):
            for i in range(0, n_each, 37):
                srv.enqueue(np.ascontiguousarray(Q[i:i + 37]), tag0=tag0 + i)
        th = [threading.Thread(target=prod, args=(Qa, 0)), threading.Thread(target=prod, args=(Qb, 100000))]
        for t in th:
            t.start()
        got = _drain(srv, 2 * n_each)
        for t in th:
            t.join()
        assert len(got) == 2 * n_each
        for i in range(n_each):
            np.testing.assert_array_equal(got[i][1], _expect(i, Qa[i, 0], 10, 10)[1])
            np.testing.assert_array_equal(got[100000 + i][1], _expect(100000 + i, Qb[i, 0], 10, 10)[1])


def test_emulated_stall_rejected_on_bad_handle():
    with pytest.raises(algas.AlgasError):
        _check_stall_on_null()


def _check_stall_on_null():
    import ctypes
    algas._check(algas.lib().algas_server_emulated_stall(ctypes.c_void_p(), ctypes.c_uint64(1)))
