"""NEXT-4 policy (host logic): trigger, longest-first victims, Profiler Eq. 2 fit, theta."""
import numpy as np

from paper_conf_isca_fenghzly025_b200 import policy


def test_pick_victims_brute_force():
    """The chosen set is the prefix of the (length desc, id asc) order that first covers
    `need` — checked against brute force over all orders' prefixes on small cases."""
    rng = np.random.default_rng(0)
    for _ in range(300):
        n = int(rng.integers(1, 7))
        b = rng.integers(0, 6, n)
        need = int(rng.integers(0, int(b.sum()) + 2))
        got = policy.pick_victims(b, need)
        order = sorted(range(n), key=lambda r: (-b[r], r))
        order = [r for r in order if b[r] > 0]
        want, s = [], 0
        for r in order:
            if s >= need:
                break
            want.append(r)
            s += b[r]
        assert got == want
        # longest first: every chosen request is at least as long as every unchosen one
        # (among positive lengths) unless the deficit was already covered
        rest = [r for r in range(n) if r not in got and b[r] > 0]
        if got and rest and sum(b[got]) < need:
            assert min(b[got]) >= max(b[rest])


def test_trigger_thresholds():
    assert policy.should_reschedule(40, 1000, 10)      # < 5 %
    assert not policy.should_reschedule(60, 1000, 10)
    assert policy.should_reschedule(60, 1000, 64)      # not enough for the next step


def test_fit_recovers_eq2():
    """Eq. 2: synthetic T = a * sumL + c with noise is recovered."""
    rng = np.random.default_rng(1)
    x = np.array([4096, 8192, 16384, 32768, 65536], float)
    y = 3e-4 * x + 2.5 + rng.normal(0, 0.01, x.size)
    a, c, r2 = policy.fit_decode_profile(x, y)
    assert abs(a - 3e-4) < 2e-6 and abs(c - 2.5) < 0.05 and r2 > 0.999


def test_theta_closed_form():
    # 1 ms step at 500 GB/s over 40 layers x 160 KiB chunks: 5e8 B / 13,107,200 B = 38.1
    assert policy.theta_from_profile(0.0, 1.0, 0, 500.0, 40, 163840) == 38
    assert policy.theta_from_profile(0.0, 0.0, 0, 500.0, 40, 163840) == 1
