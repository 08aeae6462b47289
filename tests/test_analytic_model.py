"""NEXT-4: the paper's analytic model (Eqs. 2-8) re-derived for tcgen05
(tools/analytic_model.py), checked on CPU: Eq. 4's closed form, the resource constraints of
every implemented config, and its quality as a prior against the committed measured sweep
(profiles/r01_tune_sweep_log.json)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import analytic_model as am  # noqa: E402
import tune_sweep  # noqa: E402

LOG = os.path.join(ROOT, "profiles", "r01_tune_sweep_log.json")


def test_eq4_intensity_closed_form():
    # Eq. 4: 8 bm bn bk / (4 (bm + bn) bk) = 2 bm bn / (bm + bn), independent of bk
    assert am.intensity(128, 128) == 128.0      # the paper's T4 choice (Table 4)
    assert am.intensity(256, 256) == 256.0
    assert abs(am.intensity(256, 128) - 2 * 256 * 128 / 384) < 1e-12
    # symmetric, and increasing in each argument
    assert am.intensity(64, 256) == am.intensity(256, 64)
    assert am.intensity(256, 256) > am.intensity(256, 128) > am.intensity(128, 128)


def test_every_implemented_config_fits_the_budgets():
    for cfg in tune_sweep.CONFIGS:
        g = am.geometry(cfg)
        assert am.feasible(cfg), (cfg, g)
        assert g["smem"] <= 227 * 1024 and g["tmem"] <= 512
    # a 4-stage 256x256 pair tile of hi/lo would not fit: the reason for 3 stages
    g = am.geometry((2, 256, 0, 64, 0))
    assert g["smem"] * 4 // 3 > 227 * 1024


def test_model_as_sweep_prior():
    log = json.load(open(LOG))
    res = am.evaluate(log)
    assert res["buckets"] >= 50
    # pruning the sweep to the model's top 3 keeps every bucket within a few % of the best
    assert res["top3_hit"] >= 0.85, res["top3_hit"]
    assert res["max_regret_top3"] <= 1.06, res["max_regret_top3"]
    assert res["median_regret_top1"] <= 1.01


def test_model_predicts_wave_quantisation():
    eta, conv = am.calibrate(json.load(open(LOG)))
    cfg = (2, 256, 0, 256, 0)
    # 74 pair slots: 74 tiles take one wave of MMAs, 75 take two; from 75 to 148 tiles only
    # the separate A split grows (8 B per element at the split's HBM rate)
    t74 = am.predict(cfg, 256 * 74, 256, 8192, eta, conv)
    t75 = am.predict(cfg, 256 * 75, 256, 8192, eta, conv)
    t148 = am.predict(cfg, 256 * 148, 256, 8192, eta, conv)
    wave = 3 * 128 * 256 * 8192 / am.MAC_PER_CLK / eta[am.family(cfg)] / am.F_CLK
    assert abs((t75 - t74) - wave) < 0.1 * wave
    split_delta = 8.0 * 256 * 73 * 8192 / (am.BW_HBM * am.SPLIT_EFF)
    assert abs((t148 - t75) - split_delta) < 0.05 * split_delta
