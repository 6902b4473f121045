import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) and the CUDA extension")
    import __graft_entry__ as ge
    ge.build_oracle()


@pytest.fixture(scope="session")
def graph_sets():
    """Seeded graph sets, generated once per session."""
    from workloads import make_graph_set
    cache = {}

    def get(name, **kw):
        key = (name, tuple(sorted(kw.items())))
        if key not in cache:
            cache[key] = make_graph_set(name, **kw)
        return cache[key]
    return get
