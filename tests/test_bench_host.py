"""Host logic of bench.py's clock sampler (no GPU, no nvidia-smi): which
samples count as "during the timed region" and how throttle reasons are read."""
import os
import sys
import tempfile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402

ROW = "0, {sm}, 1965, 900.0, 0x0, Not Active, Not Active, Not Active, {cap}\n"


def _sampler(lines, n0, live=True):
    fd, path = tempfile.mkstemp(suffix=".csv")
    with os.fdopen(fd, "w") as f:
        f.writelines(lines)
    s = bench.ClockSampler(0)
    s.path, s.n0, s.proc = path, n0, (object() if live else None)
    return s


def test_samples_during_region_only():
    lines = [ROW.format(sm=1000, cap="Not Active"),           # idle, before the region
             ROW.format(sm=1965, cap="Not Active"),
             ROW.format(sm=1700, cap="Active")]
    out = _sampler(lines, n0=1).summary()
    assert out["samples"] == 2 and "note" not in out
    assert out["sm_mhz"] == (1965 + 1700) / 2
    assert out["reasons"] == ["sw_power_cap"]


def test_short_region_uses_bracketing_samples_and_says_so():
    out = _sampler([ROW.format(sm=1965, cap="Not Active")], n0=1).summary()
    assert out["samples"] == 1 and out["sm_mhz"] == 1965 and "note" in out


def test_no_sampler():
    out = _sampler([], n0=0, live=False).summary()
    assert out["sm_mhz"] is None and out["reasons"] == ["nvidia-smi unavailable"]
