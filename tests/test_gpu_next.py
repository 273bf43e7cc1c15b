"""GPU parity for the §8(f) next rows (config 5): GPU-issued madvise + getrusage + pread of
/proc/self/statm on an AMR-style mesh, and rt_sigqueueinfo from a signal-search kernel."""
import numpy as np
import pytest
import torch

import inputs
import oracle
from oracle import plan
from paper_conf_isca_veselybblor18_b200 import gsys as G
from paper_conf_isca_veselybblor18_b200 import workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def gsys_instance():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    W.ensure_init()
    yield


@pytest.mark.parametrize("gflags", [G.WG | G.NONBLOCKING | G.RELAXED, G.WG | G.BLOCKING | G.RELAXED,
                                    G.WG | G.BLOCKING | G.STRONG])
def test_amr_madvise_releases_exactly_the_coarsened_blocks(gflags):
    lv = inputs.amr_levels(6, 96)
    bs = 64 << 10
    released, rss, maxrss, mesh, rc = W.amr_run(lv, block_bytes=bs, watermark_bytes=0, gflags=gflags)
    assert rc == 0
    want = plan.amr_released(lv)
    assert released.tolist() == want
    assert any(want) and not all(want)
    view = mesh.view().reshape(lv.shape[1], bs)
    for b, t in enumerate(want):
        if t:
            assert not view[b].any(), b          # MADV_DONTNEED on private anonymous memory -> zero pages
        else:
            assert (view[b] == 0xA5).all(), b
    assert (rss > 0).all() and (maxrss > 0).all()


def test_amr_watermark_gates_release():
    lv = inputs.amr_levels(4, 64, seed=11)
    released, rss, maxrss, mesh, rc = W.amr_run(lv, watermark_bytes=1 << 50)
    assert rc == 0 and not released.any()
    assert (mesh.view() == 0xA5).all()


@pytest.mark.parametrize("gflags", [G.WG | G.NONBLOCKING, G.WG | G.BLOCKING | G.RELAXED])
def test_signal_search_counts_and_ids(gflags):
    nb, bs = 512, 32 << 10
    data = inputs.signal_blocks(nb, bs)
    d = torch.from_numpy(data).cuda()
    key = inputs.dictionary()[0]
    counts, got, ts, rc = W.signal_search_run(d, nb, bs, key, gflags=gflags)
    assert rc == 0
    assert sorted(got) == list(range(nb))                  # every work-group signalled exactly once
    want = [oracle.count_key(data[b * bs:(b + 1) * bs], key) for b in range(nb)]
    assert counts.tolist() == want
    assert sum(want) > 0


# ---------------------------------------------------------------------------- config 4: memcached
@pytest.mark.parametrize("gflags,send", [(G.WG | G.BLOCKING | G.RELAXED, None), (G.WG | G.BLOCKING | G.STRONG, None),
                                         (G.WG | G.BLOCKING | G.RELAXED, G.WG | G.NONBLOCKING | G.RELAXED)])
def test_memcached_gpu_server_matches_definition(gflags, send):
    from inputs import mc as MC
    from oracle import mc as OM
    keys, vals = MC.dataset(4000, vlen=(64, 4096))
    reqs = MC.requests(keys, 5000)
    pkts = [MC.encode_get(i, k) for i, k in enumerate(reqs)]
    resp, lat, secs, stats = W.mc_serve_run(keys, vals, pkts, nwg=8, nbuckets=16, bucket_cap=1024, gflags=gflags,
                                            send_gflags=send)
    table = dict(zip(keys, vals))
    bad = [i for i, (p, r) in enumerate(zip(pkts, resp)) if r != OM.expected_response(p, table)]
    assert not bad, (len(bad), bad[:5])
    assert stats[0] == len(pkts) and stats[1] == sum(1 for k in reqs if k not in table)


def test_memcached_more_work_groups_than_service_threads():
    """48 work-groups blocked in recvfrom at once (> the service threads): empty-socket calls are
    parked by the service instead of holding a thread (reading B11); every reply stays exact."""
    from inputs import mc as MC
    from oracle import mc as OM
    keys, vals = MC.dataset(2000, vlen=(64, 1024))
    reqs = MC.requests(keys, 4000)
    pkts = [MC.encode_get(i, k) for i, k in enumerate(reqs)]
    resp, lat, secs, stats = W.mc_serve_run(keys, vals, pkts, nwg=48, nbuckets=16, bucket_cap=512,
                                            client_threads=8, window=8)
    table = dict(zip(keys, vals))
    assert all(r == OM.expected_response(p, table) for p, r in zip(pkts, resp))
    assert stats[0] == len(pkts)


def test_recvfrom_blocks_until_the_socket_timeout():
    """No traffic: every GPU recvfrom on the SO_RCVTIMEO = 20 ms socket blocks (parked on the host)
    and returns -EAGAIN once the timeout passes -- 4 work-groups x 0.3 s => at most ~60 returns,
    and at least ~ (0.3 s / 20 ms - 1) per work-group."""
    from inputs import mc as MC
    keys, vals = MC.dataset(100, vlen=64)
    resp, lat, secs, stats = W.mc_serve_run(keys, vals, [], nwg=4, nbuckets=4, bucket_cap=64, idle_s=0.3)
    assert stats[0] == 0
    assert 4 * 10 <= stats[3] <= 4 * 17, stats


# ---------------------------------------------------------------------------- row f3: Fig. 8
@pytest.mark.parametrize("gflags", [G.WG | G.BLOCKING | G.STRONG, G.WG | G.NONBLOCKING | G.STRONG,
                                    G.WG | G.BLOCKING | G.RELAXED, G.WG | G.NONBLOCKING | G.RELAXED])
@pytest.mark.parametrize("iters", [1, 5])
def test_perm_pwrite_file_equals_cpu_permutation(tmpdir_shm, gflags, iters):
    import os
    nb, bs = 300, 8192
    data, perm = inputs.perm_inputs(nb, bs)
    path = os.path.join(tmpdir_shm, f"perm_{gflags}_{iters}.bin")
    secs, rc = W.perm_pwrite_run(data, perm, iters, path, gflags, bs, grid=148)
    assert rc == 0
    got = np.fromfile(path, dtype=np.uint8)
    assert np.array_equal(got, plan.permuted_blocks(data, perm, iters, bs))


@pytest.mark.parametrize("where", ["host", "device"])
def test_poll_storm_observes_stores(where):
    """Row f4 (Fig. 9, PAPER.md:28 P28.7-11): GPU threads polling lines with system-scope loads
    keep polling for the requested time and observe a store the host makes during the storm (the
    visibility the completion polls of a5 rely on; device lines: polls counted, nothing written)."""
    import threading
    import time
    n = 64
    lines = (torch.zeros(n * 8, dtype=torch.int64).pin_memory() if where == "host"
             else torch.zeros(n * 8, dtype=torch.int64, device="cuda"))
    sink = torch.zeros(2, dtype=torch.int64, device="cuda")
    s = torch.cuda.Stream()
    nthreads = 148 * 64
    t0 = time.perf_counter()
    assert G.lib().gsys_poll_storm(lines.data_ptr(), n, nthreads, int(300e6), sink.data_ptr(), s.cuda_stream) == 0
    time.sleep(0.1)
    if where == "host":
        lines[::8] = 7                                       # plain host stores into pinned memory
    s.synchronize()
    dt = time.perf_counter() - t0
    polls, seen = int(sink[0]), int(sink[1])
    assert seen == (7 if where == "host" else 0), seen
    assert polls >= nthreads and 0.25 < dt < 5, (polls, dt)
