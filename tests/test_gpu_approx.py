"""f4 approximate mode on the GPU (128-bit fingerprints, two 64-bit
values with different radixes and primes, no base comparison) against the oracle's
approximate mode (oracle.overlaps_approx: Algorithm 2 on the P_l / S_l lists keyed by the
fingerprint pair), element by element."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import readgen

gpu = pytest.mark.gpu


def _np(t, dt):
    return t.cpu().numpy().view(dt)


@gpu
@pytest.mark.parametrize("env", [{}, {"LASAGNA_TEST_FP_BITS": "6"}, {"LASAGNA_PATH": "exact"},
                                 {"LASAGNA_TEST_LEVELS": "3", "LASAGNA_TEST_LAST_BITS": "2"}])
def test_approx_overlaps_cfg1(monkeypatch, env):
    """cfg1 reads; the stored-key hook keeps 6 fingerprint bits so that most bucket hits are
    false and must be rejected by the fingerprint pair alone; the exact LSD path and the
    three-level geometry run the same acceptance."""
    import torch
    import paper_conf_ipps_goswamilsp18_b200 as lz
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    cfg = readgen.CONFIGS["cfg1"]
    reads = readgen.config_reads(cfg)
    epl, epa, epb = oracle.overlaps_approx(reads, cfg.l_min)
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    pl, pa, pb = lz.overlaps(packed, cfg.n, cfg.L, cfg.l_min, approx=True)
    assert np.array_equal(_np(pl, np.uint8), epl)
    assert np.array_equal(_np(pa, np.uint32), epa) and np.array_equal(_np(pb, np.uint32), epb)


@gpu
@pytest.mark.parametrize("L,l_min,n,G,p_err", [(150, 90, 40_000, 300_000, 0.01),
                                             (64, 20, 30_000, 100_000, 0.0)])
def test_approx_overlaps_other_shapes(L, l_min, n, G, p_err):
    """150 bp reads (five packed words) and error-free 64 bp reads with short overlaps."""
    import torch
    import paper_conf_ipps_goswamilsp18_b200 as lz
    reads = readgen.reads(3, G, n, L, p_err)
    epl, epa, epb = oracle.overlaps_approx(reads, l_min)
    pl, pa, pb = lz.overlaps(lz.load_reads(torch.from_numpy(reads).cuda()), n, L, l_min, approx=True)
    assert len(epl) > 1000
    assert np.array_equal(_np(pl, np.uint8), epl)
    assert np.array_equal(_np(pa, np.uint32), epa) and np.array_equal(_np(pb, np.uint32), epb)
