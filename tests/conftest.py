import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) and the built CUDA extension")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture
def tuning():
    """skycube_set_tuning overrides for one test (performance-only knobs: K3 design / mode / tasks per CTA,
    device sharing), reset afterwards."""
    import paper_conf_sigmod_boghcsa17_b200 as sky

    def set_(key, value):
        sky.set_tuning(key, value)

    yield set_
    sky.set_tuning("reset", 0)
