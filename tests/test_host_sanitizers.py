"""The host-side PDL reader, model and mapper built with AddressSanitizer and
UndefinedBehaviorSanitizer and driven by tests/cpp/host_sanitize.cpp
(mutated descriptors, mapper sweep).  CPU only."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_ipps_sandrieserbp11_b200", "csrc")


@pytest.mark.skipif(shutil.which("g++") is None, reason="needs g++")
def test_host_code_under_asan_ubsan(tmp_path):
    exe = str(tmp_path / "host_sanitize")
    srcs = [os.path.join(CSRC, f) for f in ("pdl_xml.cpp", "pdl_model.cpp", "pdl_map.cpp")]
    cmd = ["g++", "-std=c++17", "-O1", "-g", "-fsanitize=address,undefined", "-fno-sanitize-recover=undefined",
           "-fno-omit-frame-pointer", "-I", CSRC, os.path.join(ROOT, "tests", "cpp", "host_sanitize.cpp"), *srcs,
           "-o", exe]
    subprocess.check_call(cmd)
    seeds = [os.path.join(ROOT, "tests", "golden", "listing1.xml"), os.path.join(ROOT, "tests", "golden", "listing2.xml"),
             os.path.join(ROOT, "paper_conf_ipps_sandrieserbp11_b200", "descriptors", "b200_x8.xml")]
    env = dict(os.environ, ASAN_OPTIONS="detect_leaks=1:abort_on_error=1", UBSAN_OPTIONS="print_stacktrace=1")
    r = subprocess.run([exe, *seeds], capture_output=True, text=True, timeout=600, env=env)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert "plans checked" in r.stdout
