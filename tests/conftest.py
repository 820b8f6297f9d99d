import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200); parity tests through the C ABI")
    config.addinivalue_line("markers", "slow: long-running (full-size configs)")
    # Build the native artefacts in-tree if they are missing (make is incremental).
    need = [os.path.join(ROOT, p) for p in ("gen/libfgrgen.so", "oracle/liboracle.so",
                                            "paper_conf_date_liulzclly22_b200/libfastgr.so")]
    if not all(os.path.exists(p) for p in need):
        subprocess.run(["make", "-C", ROOT, "-j8"], check=False, stdout=subprocess.DEVNULL)
