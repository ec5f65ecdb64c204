"""bench.py's JSON-line contract on the CPU-only reference arm (the oracle timed on the full rows,
the trees it actually ran reported as `steps`), and that non-zero ranks of a multi-rank reference
run exit without work."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(extra_env=None, extra=()):
    env = dict(os.environ)
    env.update(extra_env or {})
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "C1",
                        "--steps", "3", "--warmup", "1", "--ref-trees", "2", *extra],
                       capture_output=True, text=True, env=env, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr
    return r.stdout


def test_reference_arm_line():
    out = _run()
    d = json.loads(out.strip().splitlines()[-1])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "config", "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["higher_is_better"] is False and d["unit"] == "s/tree"
    assert d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["config"]["workload"] == "C1" and d["config"]["trees_timed"] == 3
    assert d["steps"] == 2 and d["steps_requested"] == 3          # the trees the oracle actually ran
    assert len(d["cpu_baseline"]["tree_s"]) == 2 and "full rows (1000 x 8" in d["cpu_baseline"]["sample"]


def test_reference_arm_depth_reaches_the_oracle():
    d = json.loads(_run(extra=("--depth", "2")).strip().splitlines()[-1])
    assert d["config"]["max_depth"] == 2 and "at depth 2" in d["cpu_baseline"]["sample"]


def test_reference_arm_nonzero_rank_is_silent():
    assert _run({"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"}).strip() == ""
