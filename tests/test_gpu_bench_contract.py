"""bench.py keeps the driver's contract (-m gpu): one JSON line with the required keys, a
roofline object, clock samples, an e2e object with its byte counts, and launches of our kernels;
the reference arm prints its own line.  Run on a 5% Netflix-shaped set to stay short."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(*args, timeout=600):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT,
                       capture_output=True, text=True, timeout=timeout)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [x for x in r.stdout.strip().splitlines() if x.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_json_line_contract():
    d = _bench("--steps", "3", "--warmup", "3", "--fraction", "0.05", "--e2e-steps", "1",
               "--cpu-sample", "20000")
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
                "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config",
                "roofline", "clocks", "e2e", "gpu_launches", "cpu_baseline", "deterministic"):
        assert key in d, key
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3 and d["value"] > 0
    assert d["higher_is_better"] is True and d["data"] == "synthetic"
    assert "workload" in d["config"]
    rf = d["roofline"]
    assert rf["bound"] == "hbm" and rf["unit"] == "GB/s" and rf["peak"] > 0
    assert abs(rf["frac"] - rf["achieved"] / rf["peak"]) < 1e-9
    assert d["clocks"]["sm_mhz"] > 0 and "reasons" in d["clocks"]
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert d["gpu_launches"] > 0
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == 1 and cb["value"] > 0
    assert d["deterministic"]["roofline"]["frac"] > 0
    for extra in ("grouped", "row_blocks", "row_blocks_grouped", "q_l2_only"):
        assert d[extra]["value"] > 0 and d[extra]["exactly_once_bad_units"] == 0, extra
    assert d["row_blocks"]["grid_a"] >= 1
    assert d["config"]["q_loads"].startswith("L1")          # q_cache = 0 default (R28)
    assert d["q_l2_only"]["schedule"].startswith("hogwild, q_v loads through L2")


def test_bench_hugewiki_one_gpu_uses_the_papers_64x1_blocks():
    """--workload hugewiki at N = 1 runs the paper's own blocking (i x j = 64 x 1)."""
    d = _bench("--workload", "hugewiki", "--steps", "3", "--warmup", "3", "--fraction", "0.01",
               "--no-e2e", "--cpu-sample", "20000", "--no-deterministic")
    assert d["config"]["grid_a"] == 64 and d["config"]["grid"] == "a x 1 row blocks"
    assert d["exactly_once"]["bad_units"] == 0 and d["value"] > 0


def test_bench_reference_arm_line():
    d = _bench("--impl", "reference", "--steps", "1", "--warmup", "3", "--fraction", "0.05",
               "--cpu-sample", "20000")
    assert d["impl"] == "reference" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0


@pytest.mark.parametrize("ranks", [2, 4])
def test_bench_multirank_path_emulated(ranks):
    """bench.py's N > 1 code path (Hugewiki-shaped DSGD strata, configs[3]) with N ranks as
    threads on one GPU over the library's loopback transport: the JSON line of N GPUs with its
    e2e (out-of-core epochs, H2D counted over all ranks), cpu_baseline, exactly-once record and
    the device-counted updates adding up to N per epoch -- so the first real multi-GPU run
    cannot die on a bench bug."""
    d = _bench("--emulate-ranks", str(ranks), "--steps", "3", "--warmup", "3", "--fraction", "0.002",
               "--e2e-steps", "1", "--cpu-sample", "20000")
    assert d["n_gpus"] == ranks and d["scaling"] == "strong"
    assert d["config"]["workload"].startswith("hugewiki") and d["config"]["grid_a"] == 8
    assert d["config"]["parallelism"] == f"dsgd-strata{ranks}"
    assert d["config"]["group_cols"] is True and d["config"]["batch_f"] == 1024
    eo = d["exactly_once"]
    assert eo["bad_units"] == 0 and eo["updates_per_epoch"] == eo["N"] == d["config"]["N_train"]
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0
    assert d["e2e"]["d2h_bytes_per_step"] == 8 * ranks
    assert d["cpu_baseline"]["kind"] == "oracle" and d["gpu_launches"] > 0
    assert d["emulated_ranks"]["ranks"] == ranks
    assert d["test_rmse"] < d["test_rmse_init"]
