"""Host logic of bench.py that the timing rules depend on (no GPU): the
clock / throttle summary the JSON line carries under "clocks"."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def test_clocks_summary_median_max_and_reason_union():
    c = bench.Clocks(0)
    c.nvml = object()   # rows as the NVML sampler records them
    c.rows = [(1965.0, 1965.0, set()), (1800.0, 1965.0, {"sw_power_cap"}), (1900.0, 1965.0, {"sw_power_cap"})]
    s = c.summary()
    assert s["sm_mhz"] == 1900.0 and s["sm_max_mhz"] == 1965.0
    assert s["reasons"] == ["sw_power_cap"] and s["samples"] == 3 and s["source"] == "nvml"


def test_clocks_summary_reports_rejecting_reasons():
    c = bench.Clocks(0)
    c.rows = [(1200.0, 1965.0, {"hw_thermal_slowdown"}), (1300.0, 1965.0, {"sw_thermal_slowdown", "hw_slowdown"})]
    assert c.summary()["reasons"] == ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"]


def test_clocks_unsampled_without_a_gpu():
    with bench.Clocks(0) as c:
        pass
    if not c.rows:   # no NVML / nvidia-smi here: the line says so instead of inventing clocks
        assert c.summary() == {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
