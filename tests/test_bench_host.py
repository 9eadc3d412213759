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


def test_ncu_byte_units_are_per_metric():
    """ncu prints every metric in its own unit: a Gbyte read plus a Mbyte write
    (profiles/r49_jvp: 14.76 Gbyte + 338.40 Mbyte) is 15.10e9 B, not 353e9 B
    (the r1 bug: the read's unit applied to both)."""
    import importlib.util
    import os
    spec = importlib.util.spec_from_file_location(
        "ncu_summary", os.path.join(os.path.dirname(bench.__file__), "scripts", "ncu_summary.py"))
    ns = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(ns)
    d = {"dram__bytes_read.sum": ("14.76", "Gbyte"), "dram__bytes_write.sum": ("338.40", "Mbyte")}
    assert abs(ns.dram_bytes(d) - 15.0984e9) < 1e3
    d = {"dram__bytes_read.sum": ("1,234.5", "Kbyte"), "dram__bytes_write.sum": ("7", "byte")}
    assert ns.dram_bytes(d) == 1234500.0 + 7.0
    import pytest
    with pytest.raises(ValueError):
        ns.to_bytes("1", "furlong")


def test_traffic_entries_are_keyed_to_this_build_and_plausible():
    """profiles/traffic.json: bench.py reports an entry only when its source
    revision is this build's; every entry of this build is within [0.95, 1.10] of
    the algorithmic bytes of its launch (DESIGN §6 byte model), so a unit slip or a
    stale capture cannot reach a bench line."""
    import json
    import os
    from paper_conf_sc_antepara0cw24_b200 import build as B
    sizes = bench.MESH_SIZES
    tp = os.path.join(os.path.dirname(bench.__file__), "profiles", "traffic.json")
    tr = json.load(open(tp))
    rev = B.source_rev()
    for key, e in tr.items():
        assert "rev" in e and "tag" in e, key
        cfg, elem, op, geo = key.split(":")
        if e["rev"] != rev or op not in ("jacobian", "resid", "jvp", "jvp_y") or cfg not in sizes:
            continue
        cells, nodes = sizes[cfg]
        algo = bench.bytes_per_launch(elem, cells, nodes, geo, op)
        assert 0.95 <= e["dram_bytes_per_launch"] / algo <= 1.10, (key, e["dram_bytes_per_launch"] / algo)
        got, src = bench.lookup_traffic(cfg, elem, op, geo, 1)
        assert got == e["dram_bytes_per_launch"] and e["tag"] in src
    # a stale or foreign entry is never reported
    assert bench.lookup_traffic("C4", "hex8", "jacobian", "stored", 2)[0] is None


def test_gpus_n_relaunch_refuses_without_enough_gpus(monkeypatch, capsys):
    """`python bench.py --gpus N` without a torchrun environment re-launches itself with N
    ranks, one per GPU (r1 verdict: it timed one GPU and reported n_gpus = 1); with fewer
    visible GPUs than N (and the NCCL backend) it refuses instead of oversubscribing."""
    import torch
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setenv("STOKESFO_BENCH_BACKEND", "nccl")
    monkeypatch.setattr(torch.cuda, "device_count", lambda: 1)
    assert bench.relaunch(2) == 2
    assert "needs 2 visible GPUs" in capsys.readouterr().err
    # under torchrun, --gpus must equal WORLD_SIZE
    monkeypatch.setenv("WORLD_SIZE", "3")
    monkeypatch.setenv("RANK", "0")
    monkeypatch.setattr("sys.argv", ["bench.py", "--gpus", "2", "--no-cpu-baseline"])
    assert bench.main() == 2
    assert "WORLD_SIZE = 3" in capsys.readouterr().err


def test_global_fill_byte_model_packed(monkeypatch):
    """--op jac_global byte model (DESIGN §6 NEXT-2): the element matrices are written once and read once by
    the pull assembly; in the symmetric block-packed form that is N(N+1)/2 blocks of 4 doubles per cell instead
    of (2N)^2 doubles (hex8 1,152 vs 2,048 B; wedge6 672 vs 1,152 B), everything else unchanged."""
    for elem, N in (("hex8", 8), ("wedge6", 6)):
        full = bench.bytes_per_launch(elem, 1000, 900, "stored", "jac_global", 5000)
        packed = bench.bytes_per_launch(elem, 1000, 900, "stored", "jac_global", 5000, packed=True)
        assert full - packed == 1000 * 2 * 8 * ((2 * N) ** 2 - 4 * N * (N + 1) // 2)
    # which kernels a line names: tensor cores for hex8 by default, packed global fill on them too
    monkeypatch.delenv("STOKESFO_JAC_MMA", raising=False)
    assert bench.jac_mma("hex8", "stored") and not bench.jac_mma("wedge6", "stored")
    assert bench.jac_mma("wedge6", "compact", packed=True) and bench.jac_mma("hex8", "on_the_fly")
    assert bench.kernel_name("hex8", "on_the_fly", "jacobian").startswith("eval_otf_mma_kernel<Hex8>")
    assert bench.kernel_name("hex8", "compact", "jacobian").startswith("eval_compact_mma_kernel<Hex8>")
    monkeypatch.setenv("STOKESFO_JAC_MMA", "0")
    assert not bench.jac_mma("hex8", "stored", packed=True)
    assert bench.kernel_name("hex8", "stored", "jacobian").startswith("eval_kernel<Hex8,M_JAC>")
