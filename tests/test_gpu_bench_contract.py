"""bench.py's JSON line keeps the driver contract (task statement): the DEFAULT run (every
section) on one GPU prints exactly one compact JSON line (<= 3.5 KB, strict JSON) as its last
stdout line, with the required keys; the reference arm likewise."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line(args, timeout=1500):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, cwd=ROOT,
                         capture_output=True, text=True, timeout=timeout)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = out.stdout.splitlines()
    assert lines, out.stderr[-2000:]
    last = lines[-1]
    assert len(last) <= 3500, len(last)
    assert sum(1 for x in lines if x.startswith("{")) == 1
    return json.loads(last, parse_constant=lambda c: (_ for _ in ()).throw(ValueError(c))), out


@pytest.mark.gpu
def test_bench_default_line_contract():
    j, out = _line(["--steps", "3", "--warmup", "3"])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config",
              "gpu_launches", "clocks", "roofline", "e2e", "cpu_baseline", "secondary"):
        assert k in j, k
    assert j["n_gpus"] == 1 and j["steps"] == 3 and j["warmup"] == 3
    assert j["value"] > 0 and j["gpu_launches"] > 0 and "workload" in j["config"]
    assert "CFG3" in j["config"]["workload"]
    for k in ("bound", "achieved", "peak", "unit", "frac", "traffic"):
        assert k in j["roofline"], k
    assert 0 < j["roofline"]["frac"] < 1.5
    for k in ("value", "unit", "h2d_bytes_per_step", "d2h_bytes_per_step"):
        assert k in j["e2e"], k
    assert j["e2e"]["h2d_bytes_per_step"] > 0 and j["e2e"]["value"] < j["value"]
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= set(j["clocks"])
    cb = j["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] > 0
    # every secondary section ran (a failed section is reported on stderr and has no entry)
    assert "FAILED" not in out.stderr, out.stderr[-3000:]
    for k in ("cfg3_train_bf16", "cfg2_infer_f32", "cfg2_infer_bf16", "cfg1_latency_us",
              "cfg4_epoch_bf16", "cfg5_sweep_1M_bf16", "cfg2_paper_f32", "cfg2_paper_bf16",
              "cfg2_paper_stack_train_f32"):
        assert k in j["secondary"], k
    assert j["aggregation"]["kernel"] == "gather_segsum"


def test_bench_reference_arm_contract():
    """The reference arm times the CPU oracle only: it runs here without a GPU."""
    j, _ = _line(["--impl", "reference", "--steps", "1", "--warmup", "3"], timeout=600)
    assert j["impl"] == "reference" and j["value"] > 0
    assert "CFG3" in j["config"]["workload"]
    assert j["cpu_baseline"]["kind"] == "oracle" and j["cpu_baseline"]["cores"] >= 1
    assert j["e2e"]["h2d_bytes_per_step"] == 0 and j["e2e"]["d2h_bytes_per_step"] == 0


def test_relaunch_command_is_one_rank_per_gpu():
    sys.path.insert(0, ROOT)
    import bench
    cmd = bench.relaunch_cmd(8, ["--gpus", "8", "--steps", "5"], 29511)
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=8" in cmd and "--nnodes=1" in cmd
    assert cmd[cmd.index("--master-addr") + 1] == "127.0.0.1"
    assert cmd[-3:] == ["--gpus", "8", "--steps", "5"][-3:]


def test_bench_self_calls_resolve():
    """Every self.<name>(...) call inside bench.py's Bench class names a defined method or an
    attribute assigned in the class (a removed helper otherwise only surfaces as a FAILED
    section on the GPU box)."""
    import ast
    tree = ast.parse(open(os.path.join(ROOT, "bench.py")).read())
    cls = next(n for n in tree.body if isinstance(n, ast.ClassDef) and n.name == "Bench")
    defined = {n.name for n in cls.body if isinstance(n, ast.FunctionDef)}
    assigned = set()
    for n in ast.walk(cls):
        if isinstance(n, ast.Assign):
            for t in n.targets:
                if isinstance(t, ast.Attribute) and isinstance(t.value, ast.Name) and t.value.id == "self":
                    assigned.add(t.attr)
    called = set()
    for n in ast.walk(cls):
        if (isinstance(n, ast.Call) and isinstance(n.func, ast.Attribute)
                and isinstance(n.func.value, ast.Name) and n.func.value.id == "self"):
            called.add(n.func.attr)
    missing = called - defined - assigned
    assert not missing, missing
