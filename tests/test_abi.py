"""The C-ABI library loads on a CPU host and exports every symbol include/*.h declares."""
import ctypes
import glob
import os
import re
import subprocess

from paper_conf_icppw_matzdf20_b200 import abi

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        text = open(h).read()
        text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
        for m in re.finditer(r"^[A-Za-z_][\w\s\*]*?\b(pk_\w+)\s*\(", text, flags=re.M):
            if "typedef" in text[text.rfind("\n", 0, m.start()) + 1:m.end()]:
                continue
            names.add(m.group(1))
    return names


def test_header_declares_the_north_star_calls():
    names = declared_functions()
    for n in ("pk_register_buffer", "pk_declare_affine_access", "pk_launch_partitioned", "pk_sync_to_host",
              "pk_init", "pk_enumerate", "pk_tracker_dump", "pk_timer_begin", "pk_timer_end"):
        assert n in names
    assert len(names) >= 25


def test_library_exports_every_declared_symbol():
    L = abi.lib()
    missing = [n for n in declared_functions() if not hasattr(L, n)]
    assert not missing, missing
    out = subprocess.run(["nm", "-D", "--defined-only", abi.LIB_PATH], capture_output=True, text=True).stdout
    exported = {line.split()[-1] for line in out.splitlines() if " T " in line}
    assert declared_functions() <= exported


def test_no_torch_types_in_header():
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        text = open(h).read()
        assert "torch" not in text.split("*/")[-1] and "at::" not in text and "cuda_runtime" not in text


def test_version_and_error_surface():
    assert "sm_100a" in abi.pk_version()
    L = abi.lib()
    rc = L.pk_finalize(None)
    assert rc == 0
    ctx = ctypes.c_void_p()
    rc = L.pk_init(None, ctypes.byref(ctx))
    assert rc == -1 and "null" in abi.pk_last_error()


def test_package_has_no_cpu_fallback():
    # the product package never imports the oracle
    pkg = os.path.join(ROOT, "paper_conf_icppw_matzdf20_b200")
    for py in glob.glob(os.path.join(pkg, "**", "*.py"), recursive=True):
        src = open(py).read()
        assert "import oracle" not in src and "from oracle" not in src, py
