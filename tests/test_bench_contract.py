"""The recorded bench line (profiles/r01/bench_default.json, written by `python bench.py` on a B200)
carries every key of the bench contract: the base keys, roofline (bound / achieved / peak / unit /
frac / traffic), cpu_baseline (value / unit / cores / kind / sample), e2e (value / unit / bytes per
step), clocks and gpu_launches, with no throttling reason that would void the run."""
import json
import os

import pytest

from conftest import ROOT

LINE = next((os.path.join(ROOT, "profiles", r, "bench_default.json") for r in ("r02", "r01")
             if os.path.exists(os.path.join(ROOT, "profiles", r, "bench_default.json"))), "")


@pytest.mark.skipif(not os.path.exists(LINE), reason="no recorded bench line")
def test_recorded_line_has_the_contract_keys():
    j = json.loads(open(LINE).read().strip().splitlines()[-1])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "clocks", "gpu_launches"):
        assert k in j, k
    assert j["warmup"] >= 3 and j["higher_is_better"] is True and j["scaling"] == "weak"
    assert "workload" in j["config"]
    r = j["roofline"]
    for k in ("bound", "achieved", "peak", "unit", "frac", "traffic"):
        assert k in r, k
    assert r["bound"] in ("hbm", "tensor", "alu") and 0 < r["frac"] <= 1
    assert abs(r["achieved"] / r["peak"] - r["frac"]) < 1e-6
    c = j["cpu_baseline"]
    for k in ("value", "unit", "cores", "kind", "sample"):
        assert k in c, k
    assert c["kind"] == "oracle" and (c.get("verified") or j.get("verified"))["ok"]
    e = j["e2e"]
    for k in ("value", "unit", "h2d_bytes_per_step", "d2h_bytes_per_step"):
        assert k in e, k
    assert e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert set(j["clocks"]) >= {"sm_mhz", "sm_max_mhz", "reasons"}
    assert not {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"} & set(j["clocks"]["reasons"])
    assert j["gpu_launches"] > 0
    assert {t["precision"] for t in j["per_template"]} == {"fp32", "fp32_tc", "bf16_tc"}
    for t in j["per_template"]:
        if t.get("verified") is not None:
            assert t["verified"]["ok"], t["template"]


@pytest.mark.skipif(not os.path.exists(LINE) or "r02" not in LINE, reason="no round-2 bench line")
def test_recorded_line_covers_every_config_and_measures_its_denominators():
    """Round-2 contract additions: a line per BASELINE config, each verified against
    the oracle in the run; the FP32 peak and the host link measured in the run; per-image output
    digests; overlap and bytes computed like for like; the streamed roofline of SURVEY §8(d)."""
    j = json.loads(open(LINE).read().strip().splitlines()[-1])
    cfgs = {j["config"]["baseline_config"]} | {t["baseline_config"] for t in j["per_template"]}
    assert {"configs[0]", "configs[1]", "configs[2]", "configs[3](a)", "configs[3](b)"} <= cfgs
    assert j["verified"]["ok"] and all(t["verified"]["ok"] for t in j["per_template"])
    mp = j["measured_peaks"]
    assert 60 < mp["fp32_tflops"] <= mp["fp32_unit_count_tflops_at_1965"] * 1.01
    assert j["roofline"]["peak"] == mp["fp32_tflops"]
    assert set(mp["host_link_gbs"]) == {"h2d", "d2h", "bidir_each"}
    assert j["checksum"]["digest_all"] == j["checksum"]["digest_first_share"]   # N = 1
    e = j["e2e"]
    assert 1.0 <= e["bytes_vs_lower_bound"] < 1.1
    assert e["streamed_roofline"]["bound"] in ("link", "compute") and e["streamed_roofline"]["frac"] > 0.5
    assert "uncapped" in e and e["uncapped"]["value"] > 0
    assert j["clocks"]["samples"] >= 5
