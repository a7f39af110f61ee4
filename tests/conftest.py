"""pytest configuration: the `gpu` marker and shared fixtures.

`-m "not gpu"` runs here (no GPU): oracle pins, host logic, ABI symbol checks.
`-m gpu` runs on a B200 via gpurun: parity of the CUDA path against the oracle.
"""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (sm_100a); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def oracle_mod():
    import oracle
    oracle.build()
    return oracle


@pytest.fixture(scope="session")
def inputs_mod():
    import hsort_inputs
    hsort_inputs.build()
    return hsort_inputs


@pytest.fixture(scope="session")
def hs():
    """The product binding (libhsort.so must already be built: __graft_entry__.build())."""
    import paper_conf_ipps_gowanlockk18a_b200 as hs_mod
    hs_mod.lib()
    return hs_mod


@pytest.fixture(scope="session")
def hs_gpu(hs):
    """Initialised library on a real GPU (gpu-marked tests only)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    hs.hsort_init()
    yield hs
    hs.hsort_finalize()
