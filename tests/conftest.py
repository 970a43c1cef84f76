import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")

# A fresh checkout has no libmpress.so yet: compile it (nvcc, sm_100a) before
# any test imports the binding -- compiling is not a fallback, the tests
# always run the built library.
if not (os.path.exists(os.path.join(ROOT, "paper_conf_hpca_zhouwylbyx23_b200", "libmpress.so"))
        and os.path.exists(os.path.join(ROOT, "synth", "libsynth.so"))):
    import __graft_entry__
    __graft_entry__.build()


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running test")


def pytest_collection_modifyitems(config, items):
    try:
        import torch
        have_gpu = torch.cuda.is_available()
    except Exception:  # pragma: no cover
        have_gpu = False
    if have_gpu:
        return
    skip = pytest.mark.skip(reason="no CUDA GPU in this container")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)
