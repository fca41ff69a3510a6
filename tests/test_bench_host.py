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


def test_traffic_per_step_from_profiles(tmp_path, monkeypatch):
    """roofline.traffic = the DRAM-over-algorithmic ratio of the committed ncu
    capture of one flux launch of THIS workload x the step's algorithmic bytes
    (a C5 capture may cover fewer rows than the bench's launches); absent
    workloads give None."""
    import json
    prof = tmp_path / "profiles"
    prof.mkdir()
    (prof / "ncu_flux_summary.json").write_text(json.dumps(
        {"C4": {"traffic_over_alg": 1.02, "source": "x"}, "C5": {"traffic_over_alg": 1.05}}))
    monkeypatch.setattr(bench, "ROOT", str(tmp_path))
    assert bench._traffic_from_profiles("C4", 4.6e10) == (1.02 * 4.6e10, "x")
    assert bench._traffic_from_profiles("C5", 3.1e11)[0] == 1.05 * 3.1e11
    assert bench._traffic_from_profiles("C3", 1.0) == (None, None)


def test_gpus_n_spawns_torchrun(monkeypatch):
    """`python bench.py --gpus 4` without WORLD_SIZE re-executes itself under
    torch.distributed.run with 4 ranks on 127.0.0.1."""
    calls = []
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(sys, "argv", ["bench.py", "--gpus", "4", "--steps", "2"])
    monkeypatch.setattr(bench.os, "execv", lambda exe, cmd: calls.append(cmd))
    bench.main()
    (cmd,) = calls
    assert cmd[1:3] == ["-m", "torch.distributed.run"] and "--nproc-per-node=4" in cmd
    assert cmd[cmd.index("--master-addr") + 1] == "127.0.0.1"
    assert cmd[-4:] == ["--gpus", "4", "--steps", "2"] and cmd[-5].endswith("bench.py")


def test_cpu_model_string():
    assert isinstance(bench._cpu_model(), str) and bench._cpu_model()
