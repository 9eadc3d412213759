"""Host logic of bench.py that the GPU runs depend on (no GPU needed):
the nvidia-smi clock sampler must report only samples taken inside the timed
region (the contract's 'clocks DURING the timed region'), and fall back to the
first sample after its start when the region is shorter than the sampling period."""
import datetime
import tempfile
import time

import bench


class _Proc:
    def terminate(self):
        pass

    def wait(self, timeout=None):
        pass


def _sampler(rows, t0, t1):
    c = bench.ClockSampler(0)
    c.file = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
    for ts, sm, pw, cap in rows:
        stamp = datetime.datetime.fromtimestamp(ts).strftime("%Y/%m/%d %H:%M:%S.%f")[:-3]
        c.file.write(f"{stamp}, {sm}, 1965, {pw}, 0x0, Not Active, Not Active, Not Active, "
                     f"{'Active' if cap else 'Not Active'}\n")
    c.proc = _Proc()
    c.t0, c.t1 = t0, t1
    return c


def test_clock_window_excludes_idle_samples():
    now = time.time()
    # idle at 1965 MHz before the region, capped at 1500-1600 MHz inside it, idle again after
    rows = [(now + 0.02 * k, 1965, 250, False) for k in range(10)]
    rows += [(now + 0.2 + 0.02 * k, 1500 + 20 * k, 990, True) for k in range(6)]
    rows += [(now + 0.4 + 0.02 * k, 1965, 300, False) for k in range(10)]
    out = _sampler(rows, now + 0.19, now + 0.31).stop()
    assert out["samples"] == 6
    assert 1500 <= out["sm_mhz"] <= 1600 and out["sm_min_mhz"] == 1500
    assert out["reasons"] == ["sw_power_cap"]
    assert out["power_w"] == 990
    assert out["sm_max_mhz"] == 1965


def test_clock_window_shorter_than_period_takes_next_sample():
    now = time.time()
    rows = [(now + 0.1 * k, 1965 - 100 * k, 300 + k, False) for k in range(5)]
    out = _sampler(rows, now + 0.15, now + 0.16).stop()
    assert out["samples"] == 1 and out["sm_mhz"] == 1765
