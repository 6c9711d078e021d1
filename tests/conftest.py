import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); runs the CUDA path")
    config.addinivalue_line("markers", "slow: long-running (full-size configs)")


def pytest_addoption(parser):
    parser.addoption("--ffm-lib", default=None,
                     help="run the tests against another build of libffm.so (tools/build_variants.sh)")


def pytest_sessionstart(session):
    path = session.config.getoption("--ffm-lib")
    if path:
        import paper_conf_sc_weltonm19_b200 as ffm
        ffm.set_library_path(path)
