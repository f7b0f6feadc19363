"""The device-side generator equals the numpy generator element by element."""
import numpy as np
import pytest

import wdgen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gg():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import wdgen.gpu as gg
    return gg


def _np(t):
    return t.cpu().numpy().view(np.uint32)


def test_streams_match(gg):
    n, start = 300_017, 123_456
    assert np.array_equal(_np(gg.unique_keys(n, 5, start)), wdgen.unique_keys(n, 5, start))
    assert np.array_equal(_np(gg.values(n, 6, start)), wdgen.values(n, 6, start))
    assert np.array_equal(_np(gg.uniform_keys(n, 7, start)), wdgen.uniform_keys(n, 7, start))
    assert np.array_equal(_np(gg.interleaved_queries(1000, 8, 10, 1990)),
                          wdgen.interleaved_queries(1000, 8, 10, 1990))
    import torch
    hits = torch.empty(n, dtype=torch.uint8, device="cuda")
    q = gg.mixed_queries(50_000, n, 0.5, 9, start, hits=hits)
    eq, eh = wdgen.mixed_queries(50_000, n, 0.5, 9, start)
    assert np.array_equal(_np(q), eq) and np.array_equal(hits.cpu().numpy().astype(bool), eh)


def test_zipf_stream_matches(gg):
    # rejection-inversion in float64 on both sides; libm vs libdevice may differ by 1 ulp
    # in exp/log, which can flip an accept test at a boundary: allow a 1e-5 mismatch rate
    n = 1 << 20
    a = _np(gg.zipf_keys(n, 2**32 - 1, 5, 1000))
    b = wdgen.zipf_keys(n, 2**32 - 1, 5, 1000)
    assert (a != b).mean() <= 1e-5


def test_device_closed_form_checker(gg):
    # wdgen.gpu.check_unique (used by the full-size tests) must agree with the oracle's
    # closed form: zero mismatches on the oracle's own answers, and it must count exactly
    # the answers we corrupt (a wrong value, a wrong found flag, a found absent key, a
    # not-found present key, a value written for an absent key)
    import oracle
    import torch
    n, ks, vs = 100_003, 71, 72
    q = np.concatenate([wdgen.interleaved_queries(n, ks),
                        np.array([0xFFFFFFFF], np.uint32)])
    ev, ef = oracle.expected_unique(q, n, ks, vs)
    dq = torch.from_numpy(q.view(np.int32)).cuda()
    dv = torch.from_numpy(ev.view(np.int32).copy()).cuda()
    df = torch.from_numpy(ef.copy()).cuda()
    assert gg.check_unique(dq, dv, df, n, ks, vs) == (0, None, int(ef.sum()))
    assert gg.check_unique(dq, dv, None, n, ks, vs)[0] == 0
    assert gg.check_unique(dq, None, df, n, ks, vs)[0] == 0
    hit = np.flatnonzero(ef == 1)
    miss = np.flatnonzero(ef == 0)
    dv[int(hit[5])] ^= 1                     # wrong value
    df[int(hit[9])] = 0                      # present reported absent
    df[int(miss[3])] = 1                     # absent reported present
    dv[int(miss[7])] = 0                     # absent with a value other than NOT_FOUND
    bad, first, _ = gg.check_unique(dq, dv, df, n, ks, vs)
    assert bad == 4 and first == min(hit[5], hit[9], miss[3], miss[7])
    # a different n_present moves the boundary: keys with index in [n/2, n) become absent
    assert gg.check_unique(dq, None, torch.from_numpy(ef.copy()).cuda(), n // 2, ks, vs)[0] == \
        int(((q != 0xFFFFFFFF) & (wdgen.key_index(q, ks) >= n // 2) & (wdgen.key_index(q, ks) < n)).sum())
