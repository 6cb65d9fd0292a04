import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def O():
    """The CPU oracle (test infrastructure)."""
    from oracle import oracle as mod
    mod.build()
    return mod


@pytest.fixture(scope="session")
def sk():
    from synth import skeletons
    return skeletons


@pytest.fixture(scope="session")
def paper_link(O, sk):
    rc, link = O.fit_pcie(sk.PAPER_TS, sk.PAPER_TL, sk.PAPER_SL)
    assert rc == 0
    return link
