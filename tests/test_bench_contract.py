"""The committed bench line (profiles/r1_bench_c2.json, written by bench.py on a B200) carries every key of the
driver's contract: metric/value/unit, timing, clocks, e2e with transfer bytes, launch count, roofline and the
CPU-oracle baseline.  Runs on CPU (it only parses the file)."""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line():
    txt = open(os.path.join(ROOT, "profiles", "r1_bench_c2.json")).read().strip().splitlines()[-1]
    return json.loads(txt)


def test_bench_line_contract():
    d = _line()
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "clocks", "e2e", "gpu_launches", "roofline", "cpu_baseline"):
        assert k in d, k
    assert d["metric"] == "GCUPS" and d["unit"] == "GCUPS" and d["higher_is_better"] is True
    assert d["warmup"] >= 3 and d["steps"] >= 1 and d["value"] > 0
    assert d["scaling"] == "weak" and d["data"] == "synthetic" and "workload" in d["config"]
    assert "l2" in d["config"]                                   # L2 handling between timed steps stated
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    r = d["roofline"]
    assert r["bound"] in ("alu", "hbm", "tensor") and 0 < r["frac"] <= 1
    assert abs(r["achieved"] / r["peak"] - r["frac"]) < 1e-6
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] >= 1 and c["value"] > 0 and c["sample"]
    cl = d["clocks"]
    assert cl["sm_mhz"] > 0 and not set(cl["reasons"]) & {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"}
    assert d["gpu_launches"] > 0
