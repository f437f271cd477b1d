"""-m "not gpu": the Eq. (1) fit (§IV-C, Fig. 8: measured vs predicted
migration time) on synthetic (M, T) pairs with a known alpha and beta."""
import os
import sys

import numpy as np
import pytest

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
import eq1  # noqa: E402


def test_exact_line_is_recovered():
    ms = [3 << 20, 16 << 20, 128 << 20, 1 << 30, 4 << 30]
    alpha, beta = 1 / 27e9, 0.0021  # 27 GB/s effective, 2.1 ms fixed
    ts = [alpha * m + beta for m in ms]
    a, b = eq1.fit(ms, ts)
    assert a == pytest.approx(alpha, rel=1e-9) and b == pytest.approx(beta, rel=1e-6)
    r = eq1.evaluate(ms, ts, [0, 2, 4])
    assert r["heldout_rel_err_max"] < 1e-9 and r["r2"] == pytest.approx(1.0)
    assert r["effective_GBs"] == pytest.approx(27.0, rel=1e-9)


def test_noisy_points_held_out_error_bounded():
    rng = np.random.default_rng(7)
    ms = np.geomspace(3 << 20, 8 << 30, 12)
    alpha, beta = 1 / 3.3e9, 0.05
    ts = alpha * ms + beta
    noisy = ts * (1 + rng.uniform(-0.03, 0.03, ms.size))
    r = eq1.evaluate(list(ms), list(noisy), list(range(0, 12, 2)))
    assert r["alpha_s_per_GB"] == pytest.approx(alpha * 1e9, rel=0.05)
    assert r["heldout_rel_err_max"] < 0.15  # 3 % noise on T, dominated by the small-M points


def test_tr_term_and_config_predictions():
    alpha, beta = 2e-11, 1e-3
    assert eq1.predict(alpha, beta, 1e9, tr=0.5) == pytest.approx(0.02 + 0.5 + 1e-3)
    rows = eq1.predict_configs(alpha, beta, {"C1": {"M_bytes": 3 << 20, "measured_s": 1.1e-3},
                                             "C2": {"M_bytes": 463e6, "measured_s": None}})
    assert rows[0]["rel_err"] == pytest.approx(abs(alpha * (3 << 20) + beta - 1.1e-3) / 1.1e-3)
    assert rows[1]["rel_err"] is None


def test_degenerate_inputs_rejected():
    with pytest.raises(ValueError):
        eq1.fit([1e6], [1.0])
    with pytest.raises(ValueError):
        eq1.fit([1e6, 1e6], [1.0, 2.0])
