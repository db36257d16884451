"""pytest configuration: the `gpu` marker and in-tree native builds.

`-m "not gpu"` runs here (no GPU): oracle pins, generator properties, host
logic (plan parser, cost model, merge), C-ABI symbol exports, gloo multi-rank.
`-m gpu` runs on a B200 via gpurun: CUDA-path parity against the oracle.
"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: larger-SF case")
    needed = ["tpchgen/libtpchgen.so", "oracle/liboracle.so",
              "paper_conf_sigmod_paulhh16_b200/lib/libgpl.so"]
    if any(not os.path.exists(os.path.join(ROOT, p)) for p in needed):
        subprocess.run(["make", "-s", "-j8"] + [p for p in needed if not os.path.exists(os.path.join(ROOT, p))], cwd=ROOT, check=True)
