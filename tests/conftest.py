import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")


import pytest  # noqa: E402


@pytest.fixture(autouse=True)
def _fresh_library_knobs():
    """The library caches its DDT_* knobs (ddt_reload_env): tests that set one
    with monkeypatch see it, and the next test sees it gone."""
    def reload():
        so = os.path.join(ROOT, "paper_conf_cluster_chukzsp20_b200", "libddt.so")
        if os.path.exists(so):
            try:
                from paper_conf_cluster_chukzsp20_b200 import reload_env
                reload_env()
            except Exception:
                pass
    reload()
    yield
    reload()
