import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    # The C-ABI library is a git-ignored build artefact: (re)build it in-tree when it is
    # missing or older than its sources, so a fresh checkout tests the current code.
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "_plgpu_build", os.path.join(ROOT, "paper_conf_icppw_planob21_b200", "build.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    mod.build()
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: statistical / long-running oracle pins")


def pytest_collection_modifyitems(config, items):
    if os.environ.get("PL_RUN_SLOW"):
        return
    skip = pytest.mark.skip(reason="slow pin: set PL_RUN_SLOW=1")
    for it in items:
        if "slow" in it.keywords:
            it.add_marker(skip)
