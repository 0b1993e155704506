"""The committed bench line (profiles/r2/bench_c3_j.json, written by bench.py on a B200) carries every key of the
driver's contract -- metric/value/unit, timing, clocks, e2e with transfer bytes, launch count, roofline, CPU-oracle
baseline -- on the headline config C3, and its roofline fraction can be recomputed from the line itself at the
paper's 9 ops per explored cell.  Runs on CPU (it only parses the file)."""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line():
    txt = open(os.path.join(ROOT, "profiles", "r2", "bench_c3_j.json")).read().strip().splitlines()[-1]
    return json.loads(txt)


def test_bench_line_contract():
    d = _line()
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "clocks", "e2e", "gpu_launches", "roofline", "cpu_baseline",
              "genome_pair", "secondary"):
        assert k in d, k
    assert d["metric"] == "GCUPS" and d["unit"] == "GCUPS" and d["higher_is_better"] is True
    assert d["warmup"] >= 3 and d["steps"] >= 1 and d["value"] > 0
    assert d["scaling"] == "weak" and d["data"] == "synthetic" and d["config"]["workload"].startswith("C3")
    assert "l2" in d["config"]                                   # L2 handling between timed steps stated
    assert abs(d["value"] - d["cells"] / (d["ms_per_step"] * 1e-3) / 1e9) < 1e-6 * d["value"]
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    r = d["roofline"]
    assert r["bound"] == "alu" and r["ops_per_cell"] == 9 and 0 < r["frac"] <= 1
    assert abs(r["achieved"] / r["peak"] - r["frac"]) < 1e-6
    recomputed = 9 * d["cells"] / (r["inspector_ms"] * 1e-3) / (r["peak"] * 1e12)
    assert abs(recomputed - r["frac"]) < 1e-6
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] >= 1 and c["value"] > 0 and c["sample"]
    assert c["one_core_gcups"] > 0 and c["cpu_model"] and c["gpu_speedup_vs_one_core"] > c["gpu_speedup_vs_all_cores"]
    cl = d["clocks"]
    assert cl["sm_mhz"] > 0 and not set(cl["reasons"]) & {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"}
    assert d["gpu_launches"] > 0
    g = d["genome_pair"]
    assert g["workload"].startswith("C4") and g["seeds"] == 1 << 23 and g["wall_s"] > 0
    assert d["exec_words"] <= d["exec_reserved_words"]
