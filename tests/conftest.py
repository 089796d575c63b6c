import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (CUDA path through the C ABI)")
    config.addinivalue_line("markers", "slow: long-running statistical pin")


@pytest.fixture(scope="session")
def tiny_corpus():
    from paper_conf_hpdc_xie0lt19_b200 import synth
    return synth.tiny_numpy()


@pytest.fixture(scope="session")
def tiny_cfg():
    from paper_conf_hpdc_xie0lt19_b200 import synth
    return synth.CONFIGS["tiny"]
