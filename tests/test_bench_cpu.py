"""Host logic of bench.py (CPU): how `--gpus N` is honoured, and the roofline arithmetic.

bench.py must never print a line for fewer GPUs than it was asked for: with WORLD_SIZE set it
checks it against --gpus; without a launcher it re-executes itself under torch.distributed.run
(the driver's own N > 1 launch line) or refuses when the box has fewer GPUs.
"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def test_launch_plan():
    assert bench.launch_plan(1, {}, 0) == ("run", 1)
    assert bench.launch_plan(4, {"WORLD_SIZE": "4"}, 8) == ("run", 4)
    assert bench.launch_plan(8, {}, 8) == ("relaunch", 8)
    assert bench.launch_plan(2, {}, 0, impl="reference") == ("run", 2)
    with pytest.raises(bench.LaunchError, match="needs 2 visible GPUs"):
        bench.launch_plan(2, {}, 1)
    with pytest.raises(bench.LaunchError, match="WORLD_SIZE=1"):
        bench.launch_plan(2, {"WORLD_SIZE": "1"}, 8)
    with pytest.raises(bench.LaunchError):
        bench.launch_plan(0, {}, 8)
    cmd = bench.relaunch_cmd(8, ["--gpus", "8", "--steps", "5"], 29555)
    assert cmd[1:4] == ["-m", "torch.distributed.run", "--nnodes=1"]
    assert "--nproc-per-node=8" in cmd and cmd[cmd.index("--master-addr") + 1] == "127.0.0.1"
    assert cmd[-4:] == ["--gpus", "8", "--steps", "5"] and cmd[-5].endswith("bench.py")


def test_bench_refuses_more_gpus_than_the_box_has():
    """on this GPU-less box `bench.py --gpus 2` must fail loudly, not measure one GPU"""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env["CUDA_VISIBLE_DEVICES"] = ""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"],
                       capture_output=True, text=True, env=env, timeout=600)
    assert r.returncode == 2 and "needs 2 visible GPUs" in r.stderr and r.stdout.strip() == ""


def test_primitive_roofline_bounds():
    """max-roof fractions: gathers against max(gathered / L2 peak, compulsory / HBM), GEMMs against
    max(flops / 3xTF32 roof, bytes / HBM); frac = t_roof / t"""
    l2, hbm, tc = 18000.0, 6500.0, 1386.0
    # an L2-resident gather: 90 GB gathered, 0.6 GB compulsory in 5 ms -> bound l2, 1.0
    st = {"calls": 1, "ms": 5.0, "bytes": 90e9, "flops": 0.0, "compulsory_bytes": 0.6e9, "l2_resident": 1}
    r = bench.primitive_roofline("spmm", st, hbm, tc, "measured", l2, traffic=2.0e9)
    assert r["bound"] == "l2" and abs(r["frac"] - 1.0) < 1e-9
    assert abs(r["dram"]["gbs"] - 400.0) < 1e-6 and abs(r["dram"]["frac_spec_8tbs"] - 0.05) < 1e-9
    # a streaming-bound gather: compulsory dominates -> bound hbm
    st = {"calls": 2, "ms": 2.0, "bytes": 10e9, "flops": 0.0, "compulsory_bytes": 6.5e9, "l2_resident": 0}
    r = bench.primitive_roofline("sddmm", st, hbm, tc, "measured", l2)
    assert r["bound"] == "hbm" and abs(r["frac"] - 0.5) < 1e-9 and r["launch_ms"] == 1.0
    # a GEMM above the ridge: tensor-bound against bf16 x 1/2 / 3
    st = {"calls": 1, "ms": 1.0, "bytes": 1e9, "flops": 115.5e9}
    r = bench.primitive_roofline("gemm_tc", st, hbm, tc, "measured", l2)
    assert r["bound"] == "tensor" and abs(r["frac"] - 0.5) < 1e-9
    # below the ridge: HBM-bound
    st = {"calls": 1, "ms": 1.0, "bytes": 3.25e9, "flops": 1e9}
    r = bench.primitive_roofline("gemm_tc", st, hbm, tc, "measured", l2)
    assert r["bound"] == "hbm" and abs(r["frac"] - 0.5) < 1e-9


def test_roofline_gather_beyond_l2_uses_the_dram_counter():
    """a gather whose operand exceeds L2 is bound by the DRAM traffic ncu measured, not by the
    algorithmic bytes (whose L2 hit rate is unknown)"""
    st = {"calls": 2, "ms": 10.0, "bytes": 100e9, "flops": 0.0, "compulsory_bytes": 5e9, "l2_resident": 0}
    r = bench.primitive_roofline("spmm", st, 6500.0, 1386.0, "measured", 18000.0, traffic=26e9)
    assert r["bound"] == "hbm" and abs(r["achieved"] - 5200.0) < 1e-6 and abs(r["frac"] - 0.8) < 1e-9


def test_roofline_gather_rate_bounds():
    """the K = 1 SDDMM is bound by random 4-byte gathers (one per entry: flops = 2 nnz) against the
    measured gather rate (profiles/gather_rate.json); a gather beyond L2 with no ncu traffic for its
    workload is held to the measured random-row rate"""
    gp, rp = bench.gather_peak(), bench.row_gather_peak()
    assert gp is not None and 250e9 < gp < 400e9 and rp is not None and 5000 < rp < 8000
    nnz = 130e6
    st = {"calls": 1, "ms": 1.0, "bytes": nnz * 12, "flops": 2 * nnz, "compulsory_bytes": nnz * 8,
          "l2_resident": 1}
    r = bench.primitive_roofline("sddmm", st, 6500.0, 1386.0, "measured", 18000.0)
    assert r["bound"] == "gather" and abs(r["achieved"] - 130.0) < 1e-6 and abs(r["frac"] - 130e9 / gp) < 1e-9
    st = {"calls": 1, "ms": 10.0, "bytes": 60e9, "flops": 0.0, "compulsory_bytes": 3e9, "l2_resident": 0}
    r = bench.primitive_roofline("gat_bwd_a", st, 6500.0, 1386.0, "measured", 18000.0)
    assert r["bound"] == "row_gather" and abs(r["achieved"] - 6000.0) < 1e-6 and abs(r["frac"] - 6000.0 / rp) < 1e-9
    assert abs(r["gathered"]["frac_row_gather"] - 6000.0 / rp) < 1e-9
