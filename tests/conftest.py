import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (runs through the CUDA C-ABI library)")


@pytest.fixture(scope="session")
def orc():
    import oracle
    oracle.build()
    return oracle


@pytest.fixture(scope="session")
def sess():
    """One context + queue on cuda:0 through the C-ABI (GPU tests only)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_sc_kimdjjl15_b200 import build, cl
    build.build()
    S = cl.Session(0)
    yield S
    S.close()


def pytest_terminal_summary(terminalreporter):
    """Worst LINEAR error per parity check, in fp32 ulps (reading A10)."""
    try:
        from tests.gpu_helpers import WORST
    except Exception:
        return
    if not WORST:
        return
    items = sorted(WORST.items(), key=lambda kv: -kv[1])
    terminalreporter.write_line(f"LINEAR parity: {len(items)} checks, worst {items[0][1]:.2f} ulp "
                                f"({items[0][0]}); bound 4 ulp, 1e-6 abs below 2^-10")
    for what, u in items[:10]:
        terminalreporter.write_line(f"  {u:5.2f} ulp  {what}")
