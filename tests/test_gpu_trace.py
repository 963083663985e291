"""Declared descriptors vs what the kernels touch (SURVEY.md §5 / hard part H5; P:L568-571
write maps exact, read maps may over-approximate; P:L1231-1236 a kernel clone marking the
memory it accesses).

Runs tests/trace_worker.py against libpk_trace.so (the access-recording build): for every
builtin at P = 1 and P = 3, every launch's recorded stores must EQUAL the declared write
set of each partition and its recorded fetches must lie inside the declared read set
(dilated only by the TMA over-fetch stated in tests/access_cases.py).  Whether the
over-fetched bytes influence any result is a separate question, answered by the poison
test in tests/test_gpu_access.py.
"""
import json
import os
import subprocess
import sys

import pytest

from paper_conf_icppw_matzdf20_b200 import build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def trace_results():
    build.build(trace=True)
    env = dict(os.environ, PK_TRACE_ACCESS="1")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "trace_worker.py")], env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    out = {}
    for line in r.stdout.splitlines():
        if line.startswith("{"):
            d = json.loads(line)
            out[(d["case"], d["P"])] = d
    return out


sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import access_cases as AC  # noqa: E402

RUNS = [(name, P) for name in AC.CASES for P in AC.parts(name)]


@pytest.mark.parametrize("case,P", RUNS)
def test_recorded_accesses_match_descriptors(trace_results, case, P):
    d = trace_results[(case, P)]
    assert d["stray"] == 0, d
    assert d["stored_words"] > 0 and d["fetched_words"] > 0, d
    assert not d["write_mismatch"], d["write_mismatch"][:4]
    assert not d["read_outside"], d["read_outside"][:4]
