"""The committed bench line (profiles/r2_bench.json, written by bench.py on a B200)
keeps the driver's JSON contract: every required key, the timing rules it can
show (warm-up >= 3, clocks sampled inside the timed region, no throttle reason
that rejects a run), and self-consistent derived numbers."""
import json
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LINE = os.path.join(ROOT, "profiles", "r2_bench.json")


@pytest.fixture(scope="module")
def line():
    if not os.path.exists(LINE):
        pytest.skip("no committed bench line")
    return json.loads(open(LINE).read().strip().splitlines()[-1])


def test_required_keys(line):
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert k in line, k
    assert line["unit"] == "nodes/s" and line["higher_is_better"] is True and line["scaling"] == "weak"
    assert line["data"] == "synthetic" and "workload" in line["config"]
    assert line["vs_baseline"] is None  # the paper publishes no number for this metric


def test_timing_rules(line):
    assert line["warmup"] >= 3 and line["steps"] >= 1
    assert "l2" in line["config"]  # scrub (or inputs larger than L2) stated
    clk = line["clocks"]
    assert clk and clk["samples"] >= 1 and clk["sm_mhz"] > 0.5 * clk["sm_max_mhz"]
    assert not {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"} & set(clk["reasons"])
    assert line["gpu_launches"] > 0 and line["gpu_launches"] % line["steps"] == 0


def test_derived_numbers(line):
    nodes = line["config"]["nodes_per_rank"] * line["n_gpus"]
    assert line["value"] == pytest.approx(nodes / (line["ms_per_step"] / 1e3), rel=1e-6)
    rl = line["roofline"]
    assert rl["bound"] in ("hbm", "tensor", "alu") and rl["unit"] in ("GB/s", "TFLOP/s")
    assert rl["frac"] == pytest.approx(rl["achieved"] / rl["peak"], rel=1e-9)
    assert rl["traffic"] is None or rl["traffic"] > 0
    cpu = line["cpu_baseline"]
    assert cpu["kind"] == "oracle" and cpu["cores"] >= 1 and cpu["value"] > 0 and cpu["sample"]
    e2e = line["e2e"]
    assert e2e["unit"] == line["unit"] and e2e["h2d_bytes_per_step"] > 0 and e2e["d2h_bytes_per_step"] > 0
    assert e2e["value"] < line["value"]  # the end-to-end number is not the device-timed one


def test_multi_gpu_block(line):
    mg = line["multi_gpu"]
    assert mg["collective"].startswith("none")
    assert len(mg["headline_per_rank"]) == line["n_gpus"]
    assert all(r["parity"]["ok"] for r in mg["headline_per_rank"])
    c5 = mg["c5"]
    assert len(c5["per_gpu"]) == line["n_gpus"]
    for g in c5["per_gpu"]:
        assert g["seed"] == 100 + g["rank"] and g["parity"]["ok"]
    nodes = sum(g["nodes"] for g in c5["per_gpu"])
    assert c5["aggregate_nodes_per_s"] == pytest.approx(nodes / (c5["ms_per_step"] / 1e3), rel=1e-6)


def test_whole_step_fraction(line):
    ws = line["roofline"]["whole_step"]
    assert ws["ms_per_step"] == pytest.approx(line["ms_per_step"], rel=1e-9)
    assert ws["achieved"] == pytest.approx(ws["alg_bytes"] / (ws["ms_per_step"] / 1e3) / 1e9, rel=1e-6)
