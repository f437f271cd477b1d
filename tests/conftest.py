import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    # libchecl.so is an in-tree build artefact (git-ignored): make sure it exists so the
    # ABI tests exercise the real library. nvcc cross-compiles sm_100a without a GPU.
    import __graft_entry__
    __graft_entry__._build_module().build(experiments=True)
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running")
