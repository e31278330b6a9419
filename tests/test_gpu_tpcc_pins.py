"""The hand-computed TPC-C pins of tests/test_oracle_tpcc_pins.py, run on the CUDA path through
the C-ABI (StockLevel window / threshold / distinct items, OrderStatus slots, Delivery counts,
totals and effects, the by-name customer choice, the empty-queue RAW abort).  The fixture's
CUSTOMER / ITEM / STOCK / ORDER keys are sparse, so these batches also run the PK hash-index
probes that the dense-keyed bench tables skip."""
import pytest

from tests import tpcc_tiny as tt
from tests.test_oracle_tpcc_pins import *  # noqa: F401,F403  (the same test functions)
from workloads import tpcc

pytestmark = pytest.mark.gpu


class _GpuDb:
    """The oracle's run_tpcc / dump_table interface over the CUDA path."""

    def __init__(self, mode):
        import paper_conf_icde_wei0l0lzj024_b200 as ltpg
        self.ltpg = ltpg
        wl = tpcc.TpccWorkload(1, mode=mode)
        self.tables = tt.tiny_tables()
        self.g = ltpg.tpcc_database(wl, max_txns=64, tables=self.tables, append_batches=2)

    def run_tpcc(self, batch, clock):
        try:
            out = self.g.run_tpcc(batch, clock=clock)
        except self.ltpg.LtpgError as e:
            return e.rc, None, None
        return 0, out["status"], out["reads"]

    def dump_table(self, t):
        return self.g.dump_table(t)


@pytest.fixture
def make_db():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")

    def f(mode="strict"):
        db = _GpuDb(mode)
        return db.tables, db
    return f
