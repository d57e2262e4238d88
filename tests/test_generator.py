"""Pins of the oracle's copy of the input generator (docs/GENERATOR.md):
published splitmix64 outputs, 128-bit multiply-high, the zipf CDF against the
Euler-Maclaurin closed form of the generalized harmonic number, and the
workload mixes the configs name (BASELINE.json configs)."""
import numpy as np
import pytest
import scipy.special

import oracle
from tests import _ref as R


def test_mix64_published_vector():
    # splitmix64 seeded with 0: outputs are mix64(i * golden), i = 0, 1, 2
    assert oracle.mix64(0) == 0xE220A8397B1DCDAF
    assert oracle.mix64(R.GOLDEN) == 0x6E789E6AA1B965F4
    assert oracle.mix64((2 * R.GOLDEN) & R.M64) == 0x06C45D188009454F


def test_mix64_matches_python_spelling():
    rng = np.random.default_rng(0)
    for x in rng.integers(0, 2**63, size=200, dtype=np.int64).tolist() + [0, 2**64 - 1]:
        assert oracle.mix64(x) == R.mix64(x)


def test_uniform_is_multiply_high():
    rng = np.random.default_rng(1)
    for _ in range(200):
        u = int(rng.integers(0, 2**63)) * 2 + int(rng.integers(0, 2))
        n = int(rng.integers(1, 2**32))
        assert oracle.uniform(u, n) == (u * n) >> 64
    assert oracle.uniform(2**64 - 1, 7) == 6


def test_draw_composition():
    seed, tx, k = 12345, 987654321, 3
    inner = R.mix64(seed ^ ((tx * 0xD1B54A32D192ED03) & R.M64))
    assert oracle.draw(seed, tx, k) == R.mix64((inner + k) & R.M64)


@pytest.mark.parametrize("n,theta_milli", [(4096, 990), (1000, 500), (1 << 16, 990)])
def test_zipf_cdf_closed_form(n, theta_milli):
    theta = theta_milli / 1000
    cdf = oracle.zipf_cdf(n, theta_milli)
    assert cdf[-1] == 2**64 - 1
    assert np.all(np.diff(cdf.astype(object)) >= 0)
    # H_{n,theta} by Euler-Maclaurin: zeta(theta) + n^(1-t)/(1-t) + n^-t/2 - t n^(-t-1)/12
    H = scipy.special.zeta(theta) + n ** (1 - theta) / (1 - theta) + n ** -theta / 2 \
        - theta * n ** (-theta - 1) / 12
    p = np.diff(np.concatenate([[0.0], cdf.astype(np.float64) / 2.0**64]))
    r = np.arange(1, n + 1, dtype=np.float64)
    expect = r ** -theta / H
    assert np.allclose(p[:-1], expect[:-1], rtol=1e-9, atol=1e-15)
    if (n, theta_milli) == (4096, 990):
        assert abs(p[0] - 0.1081) < 1e-3      # top account p = 10.8%


def test_zipf_pick_frequencies():
    n = 64
    cfg = oracle.bank_cfg(n, 4, dist=oracle.DIST_ZIPF, zipf_theta_milli=990, p_update_ppm=1_000_000)
    d = oracle.bank_gen(cfg, 3, 200_000)
    src = np.bincount(d["src"], minlength=n) / len(d)
    r = np.arange(1, n + 1, dtype=np.float64)
    p = r ** -0.99 / (r ** -0.99).sum()
    assert np.abs(src - p).max() < 0.01


def test_upper_bound_edges():
    cdf = np.array([10, 10, 20, 2**64 - 1], dtype=np.uint64)
    L = oracle.lib()
    ub = lambda u: L.or_upper_bound(cdf.ctypes.data, 4, u)
    assert ub(0) == 0 and ub(9) == 0 and ub(10) == 2 and ub(19) == 2 and ub(20) == 3
    assert ub(2**64 - 1) == 3


def test_bank_c1_slot_rule():
    cfg = oracle.bank_cfg(1024, 4, ro_period=10, ro_reads=0)
    d = oracle.bank_gen(cfg, 1, 11111)
    ro = np.nonzero(d["is_update"] == 0)[0]
    assert len(ro) == 1111 and np.all(ro % 10 == 9)
    assert np.all(d["len"][ro] == 1024) and np.all(d["start"][ro] == 0)


def test_bank_threshold_mix_and_fields():
    cfg = oracle.bank_cfg(1 << 20, 4, p_update_ppm=500_000, ro_reads=64)
    d = oracle.bank_gen(cfg, 1, 100_000)
    u = d["is_update"] == 1
    assert abs(u.mean() - 0.5) < 0.01
    assert np.all(d["src"][u] != d["dst"][u])
    assert d["amt"][u].min() == 1 and d["amt"][u].max() == 100
    assert np.all(d["len"][~u] == 64)
    assert abs(d["start"][~u].mean() / (1 << 20) - 0.5) < 0.01
    # uniform endpoints: chi-square-ish check over 16 buckets
    h = np.bincount(d["src"][u] >> 16, minlength=16) / u.sum()
    assert np.abs(h - 1 / 16).max() < 0.01
    # p_update = 100% / 0%
    assert oracle.bank_gen(oracle.bank_cfg(8, 2, p_update_ppm=1_000_000), 1, 1000)["is_update"].all()
    assert not oracle.bank_gen(oracle.bank_cfg(8, 2, p_update_ppm=0), 1, 1000)["is_update"].any()


def test_tx_offset_is_counter_based():
    cfg = oracle.bank_cfg(1000, 4, p_update_ppm=300_000, ro_reads=8)
    a = oracle.bank_gen(cfg, 9, 500)
    b = oracle.bank_gen(cfg, 9, 100, tx0=400)
    assert np.array_equal(a[400:], b)


# ---- the KV generator (or_kv_gen, docs/GENERATOR.md 4): pinned by the
# statistics the workload is defined by (zipf keys, a GET/PUT mix),
# not by re-typing its formulas ----
def test_kv_gen_mix_and_zipf_frequencies():
    n_keys, n = 1024, 400_000
    cfg = oracle.kv_cfg(4096, 16, n_keys=n_keys, p_update_ppm=200_000, zipf_theta_milli=990)
    d = oracle.kv_gen(cfg, 7, n)
    # PUT fraction 20 %: binomial, 5 sigma
    f = d["is_update"].mean()
    assert abs(f - 0.2) < 5 * np.sqrt(0.2 * 0.8 / n), f
    # key frequencies against the zipf pmf r^-0.99 / H (numpy, independent of the oracle's CDF)
    r = np.arange(1, n_keys + 1, dtype=np.float64) ** -0.99
    pmf = r / r.sum()
    cnt = np.bincount(d["key"], minlength=n_keys)
    assert cnt.shape[0] == n_keys  # every key < n_keys
    for k in (0, 1, 2, 9, 99):
        sd = np.sqrt(n * pmf[k] * (1 - pmf[k]))
        assert abs(cnt[k] - n * pmf[k]) < 5 * sd, (k, cnt[k], n * pmf[k])
    # GETs carry no value; PUT values are 32 uniformly random bytes
    assert not d["val"][d["is_update"] == 0].any()
    bits = np.unpackbits(d["val"][d["is_update"] == 1].view(np.uint8))
    assert abs(bits.mean() - 0.5) < 0.005


def test_kv_gen_is_counter_based():
    cfg = oracle.kv_cfg(1 << 12, 16, p_update_ppm=300_000)
    whole = oracle.kv_gen(cfg, 11, 5000)
    part = oracle.kv_gen(cfg, 11, 1000, tx0=3000)
    assert np.array_equal(whole[3000:4000], part)
    other = oracle.kv_gen(cfg, 12, 5000)
    assert (whole["key"] != other["key"]).mean() > 0.5


def test_kv_gen_uniform_keys():
    n_keys, n = 64, 200_000
    cfg = oracle.kv_cfg(1 << 10, 16, n_keys=n_keys, dist=oracle.DIST_UNIFORM, p_update_ppm=500_000)
    cnt = np.bincount(oracle.kv_gen(cfg, 3, n)["key"], minlength=n_keys)
    chi2 = ((cnt - n / n_keys) ** 2 / (n / n_keys)).sum()
    assert chi2 < 63 + 5 * np.sqrt(2 * 63), chi2  # 63 degrees of freedom
