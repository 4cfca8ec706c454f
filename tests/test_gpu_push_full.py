"""Full-size (BASELINE configs[3], 128^3 3D 27-point) single-SpMV parity of every row block of the
push-fused row partition, P = 2 / 4 / 8, every push-kernel instance (DIA at every forced diagonal
split S incl. the register-spilling fp32 S >= 2 instances, ELL, CSR stream (fp64 spills), CSR tile,
COO, HYB), per row at 1e-12 (fp64) / 1e-5 (fp32) against |A||x|, plus bitwise ghost delivery.
The work runs in tests/push_parity_worker.py (one subprocess per S: the library reads SFS_DIA_S once)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("S", ["auto", "1", "2", "4", "8", "16"])
def test_push_rowblocks_full_size_single_spmv(S):
    env = dict(os.environ)
    cmd = [sys.executable, os.path.join(ROOT, "tests", "push_parity_worker.py")]
    if S != "auto":
        env["SFS_DIA_S"] = S
        cmd += ["--formats", "DIA:-1"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    lines = [json.loads(l) for l in r.stdout.splitlines() if l.startswith("{")]
    bad = [d for d in lines if not d["ok"]]
    assert r.returncode == 0 and not bad and lines, (bad, r.stderr[-3000:])
    assert all(d["rows"] == 2097152 for d in lines)
    expect = 3 * 2 * (1 if S != "auto" else 6)
    assert len(lines) == expect, (len(lines), expect)
