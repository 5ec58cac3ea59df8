"""Full-size parity on the BASELINE configs C3 (SSSP grid), C4 (WCC RMAT-26) and C5 (PR RMAT-25 EF44, K=20),
in the launch configuration bench.py times (tools/parity_full.py). Several minutes and ~40 GB of host
memory, so it runs only with GUM_FULL_SIZE=1 (the round's evidence is profiles/round2/parity_full_*.json)."""
import os

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.mark.skipif(os.environ.get("GUM_FULL_SIZE") != "1", reason="full-size configs: set GUM_FULL_SIZE=1")
@pytest.mark.parametrize("config", ["C3", "C4", "C5"])
def test_full_size_parity(config):
    from tools import parity_full

    rec = parity_full.check(config, n_sources=2)
    assert rec["exact"], rec
