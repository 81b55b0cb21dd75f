"""bench.py's command line (CPU): the driver's flags and the documented options
parse (a typo in the argument table once took the whole bench down)."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_help_lists_the_contract_flags():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--help"],
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    for flag in ["--gpus", "--steps", "--warmup", "--impl", "--no-options", "--no-cpu-baseline",
                 "--cpu-sample", "--path", "--config"]:
        assert flag in out.stdout, flag
