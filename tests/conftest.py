import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (sm_100a) device")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def golden_dir():
    return os.path.join(ROOT, "tests", "golden")


@pytest.fixture(autouse=True)
def _gpu_tests_on_a_side_stream(request):
    """GPU tests run on a non-default torch stream, like bench.py: the library binds torch's
    current stream (Solver.use_torch_stream), so its kernels are ordered with the test's own
    torch ops and launched with programmatic dependent launch (not used on the legacy stream)."""
    if request.node.get_closest_marker("gpu") is None:
        yield
        return
    import torch
    if not torch.cuda.is_available():
        yield
        return
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        yield
    s.synchronize()
