import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a) and the built libad.so")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def cfg1():
    from paper_conf_sc_solis_vasquezts25_b200 import synth
    return synth.make_config(1)


@pytest.fixture(scope="session")
def cfg2():
    from paper_conf_sc_solis_vasquezts25_b200 import synth
    return synth.make_config(2)


@pytest.fixture(scope="session")
def cfg3():
    from paper_conf_sc_solis_vasquezts25_b200 import synth
    return synth.make_config(3)
