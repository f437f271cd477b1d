"""PAPER.md Eq. (1) (L42-L44 §IV-C): the migration time model Tm = alpha*M + Tr + beta,
M = checkpoint (image) size, Tr = recompilation time (0 for a buffer snapshot: there
are no programs to rebuild), alpha and beta fitted by least squares (DESIGN.md reading
24). Pure numpy; the measurement driver is tools/cost_model.py."""
from __future__ import annotations

import statistics
from typing import Dict, List, Sequence

import numpy as np


def fit(ms: Sequence[float], ts: Sequence[float]):
    """(alpha, beta) minimising sum (alpha*M + beta - T)^2 (Tr = 0)."""
    if len(ms) < 2 or len(set(ms)) < 2:
        raise ValueError("Eq. (1) needs at least two distinct sizes")
    A = np.vstack([np.asarray(ms, float), np.ones(len(ms))]).T
    (alpha, beta), *_ = np.linalg.lstsq(A, np.asarray(ts, float), rcond=None)
    return float(alpha), float(beta)


def predict(alpha: float, beta: float, m: float, tr: float = 0.0) -> float:
    return alpha * m + tr + beta


def evaluate(ms: Sequence[float], ts: Sequence[float], fit_idx: Sequence[int]) -> Dict:
    """Fit on fit_idx; predicted vs measured on every point, error on the held-out ones."""
    alpha, beta = fit([ms[i] for i in fit_idx], [ts[i] for i in fit_idx])
    pred = [predict(alpha, beta, m) for m in ms]
    hold = [i for i in range(len(ms)) if i not in set(fit_idx)]
    err = [abs(pred[i] - ts[i]) / ts[i] for i in hold]
    ss_res = sum((p - t) ** 2 for p, t in zip(pred, ts))
    ss_tot = sum((t - statistics.mean(ts)) ** 2 for t in ts)
    return {"alpha_s_per_GB": alpha * 1e9, "effective_GBs": (1 / alpha / 1e9) if alpha > 0 else None,
            "beta_s": beta, "r2": 1 - ss_res / ss_tot if ss_tot else None,
            "heldout_rel_err_max": max(err) if err else None,
            "heldout_rel_err_mean": statistics.mean(err) if err else None,
            "predicted_s": pred, "measured_s": list(ts)}


def predict_configs(alpha: float, beta: float, configs: Dict[str, Dict]) -> List[Dict]:
    """Predicted vs measured Tm for named configurations {name: {M_bytes, measured_s}}."""
    out = []
    for name, c in configs.items():
        p = predict(alpha, beta, c["M_bytes"])
        m = c.get("measured_s")
        out.append({"config": name, "M_bytes": c["M_bytes"], "predicted_s": p, "measured_s": m,
                    "rel_err": abs(p - m) / m if m else None})
    return out
