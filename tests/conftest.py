import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: longer CPU test")


def pytest_sessionstart(session):
    # the C-ABI library and the oracle/generator libraries are built in-tree
    # (nvcc cross-compiles for sm_100a without a GPU)
    from paper_conf_hpdc_khorasanivgb14_b200 import build as _b
    _b.build()
    import graphgen
    import oracle
    graphgen.build()
    oracle.build()
